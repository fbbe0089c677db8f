# A/B of the current tree against _ab/base (a git worktree of an older commit, built here):
# bash scripts/ab_gpu.sh OUT "configs" "env variants" reps
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/$1; mkdir -p $OUT
CFGS=${2:-c2}; VARS=${3:-"X=0"}; REPS=${4:-2}
for r in $(seq $REPS); do for c in $CFGS; do for side in base cur; do for v in $VARS; do
  if [ $side = base ]; then D=_ab/base; else D=.; fi
  (cd $D && env $v timeout 300 python bench.py --config $c --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > /tmp/b.json 2>/dev/null)
  python -c "
import json,sys; d=json.loads(open('/tmp/b.json').read().strip().splitlines()[-1]); r=d['roofline']
print('$side $c $v', round(d['value']/1e6,1), 'Mevals/s', round(d['ms_per_step'],4), 'ms', {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})" | tee -a $OUT/ab.txt
done; done; done; done
