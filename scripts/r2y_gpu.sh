cd $GRAFT_REPO_ROOT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_svr.py -x -q 2>&1 | tail -1
for side in base cur; do
  if [ $side = base ]; then D=_ab/base; else D=.; fi
  (cd $D && timeout 600 python bench.py --config c3 --models svr --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > /tmp/b.json 2>/dev/null)
  python -c "
import json; d=json.loads(open('/tmp/b.json').read().strip().splitlines()[-1]); r=d['roofline']
print('$side c3 svr', round(d['value']/1e6,1), round(d['ms_per_step'],3), r.get('svr_contraction',{}).get('frac'), {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})"
done
for v in "SYNERGY_SPLIT_PIECE=4" "SYNERGY_SPLIT_PIECE=8" "SYNERGY_SPLIT_PIECE=12" "SYNERGY_SPLIT_PIECE=16"; do for sp in "SYNERGY_TM_SPLIT=1"; do
  env $v $sp timeout 300 python bench.py --config c2 --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > /tmp/b.json 2>/dev/null
  python -c "
import json; d=json.loads(open('/tmp/b.json').read().strip().splitlines()[-1]); r=d['roofline']
print('c2 $v $sp', round(d['value']/1e6,1), round(d['ms_per_step'],4), {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})"
done; done
for v in "SYNERGY_SPLIT_PIECE=4" "SYNERGY_SPLIT_PIECE=8"; do
  env $v timeout 300 python bench.py --config c5 --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > /tmp/b.json 2>/dev/null
  python -c "
import json; d=json.loads(open('/tmp/b.json').read().strip().splitlines()[-1]); r=d['roofline']
print('c5 $v', round(d['value']/1e6,1), round(d['ms_per_step'],4), {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})"
done
