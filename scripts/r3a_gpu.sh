cd $GRAFT_REPO_ROOT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "default" 2>&1 | tail -1
for v in "SYNERGY_TM_KB=256" "SYNERGY_TM_KB=512" "SYNERGY_TM_KB=1024" "SYNERGY_TM_KB=512 SYNERGY_TM_SLAB=30720"; do for c in c3 c4; do
  env $v timeout 300 python bench.py --config $c --steps 6 --warmup 2 --no-cpu-baseline --no-e2e > /tmp/b.json 2>/dev/null
  python -c "
import json; d=json.loads(open('/tmp/b.json').read().strip().splitlines()[-1]); r=d['roofline']
print('$c $v', round(d['value']/1e6,1), round(d['ms_per_step'],3), {k:(round(v['ms_per_launch'],4),v['launches']) for k,v in r['per_kernel'].items()})"
done; done
