#!/bin/bash
# A/B of tree-major knobs on c2/c3/c5 (device-resident, no CPU baseline / e2e).  Env lists:
#   CFGS (default "c2 c5 c3"), VARS (space-separated NAME=ENV1,ENV2 entries; "base" = defaults)
OUT=gpurun_out/${1:-tmab}
mkdir -p $OUT
python -c "import paper_conf_sc_fandccfc23_b200.build as b; b.build()" > $OUT/build.log 2>&1
for c in ${CFGS:-c2 c5 c3}; do
  for v in ${VARS:-base}; do
    name=${v%%=*}; envs=${v#*=}; [ "$name" = "$v" ] && envs=""
    env ${envs//,/ } timeout 300 python bench.py --config $c --steps ${STEPS:-10} --warmup 3 --no-cpu-baseline --no-e2e > $OUT/${c}_$name.json 2> $OUT/${c}_$name.err
    python -c "
import json
try:
  d=json.load(open('$OUT/${c}_$name.json')); print('$c $name', '%.3e'%d['value'], round(d['ms_per_step'],4), {k:round(v['ms_per_launch'],4) for k,v in d['roofline']['per_kernel'].items()})
except Exception as e: print('$c $name FAIL', e, open('$OUT/${c}_$name.err').read()[-1500:])
"
  done
done
