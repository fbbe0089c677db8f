#!/bin/bash
# A/B of launch-configuration knobs on the current build (under gpurun):
#   bash scripts/ab_env.sh OUT "configs" "env variants (VAR=v,...)" reps
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/$1; mkdir -p $OUT
CFGS=${2:-c3}; VARS=${3:-"X=0"}; REPS=${4:-2}
for r in $(seq $REPS); do for c in $CFGS; do for v in $VARS; do
  env ${v//,/ } timeout 300 python bench.py --config $c --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > /tmp/b.json 2>/tmp/b.err
  python -c "
import json,sys; d=json.loads(open('/tmp/b.json').read().strip().splitlines()[-1]); r=d['roofline']
print('$c $v', round(d['value']/1e6,1), 'Mevals/s', round(d['ms_per_step'],4), 'ms', 'frac', round(r.get('frac') or 0,3), {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})" 2>&1 | tee -a $OUT/ab.txt
done; done; done
