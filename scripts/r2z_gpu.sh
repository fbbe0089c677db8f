cd $GRAFT_REPO_ROOT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_svr.py -x -q 2>&1 | tail -2
for c in c2 c3; do
  timeout 600 python bench.py --config $c --models svr --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > /tmp/b.json 2>/dev/null
  python -c "
import json; d=json.loads(open('/tmp/b.json').read().strip().splitlines()[-1]); r=d['roofline']
print('$c svr', round(d['value']/1e6,1), round(d['ms_per_step'],3), r.get('svr_contraction',{}).get('frac'), {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})"
done
