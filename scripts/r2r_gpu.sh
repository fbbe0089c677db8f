cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2r; mkdir -p $OUT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "default or tm_nobalance or tm_nt1024 or tm_split or tm_static or tm_kb32 or tm_nsub3" > $OUT/pytest.log 2>&1; tail -2 $OUT/pytest.log
for c in c2 c3 c5 c1; do for v in "SYNERGY_TM_BALANCE=0" "SYNERGY_TM_BALANCE=1" "SYNERGY_TM_NT=1024"; do
  env $v timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/b.json 2>/dev/null
  python -c "
import json,sys; d=json.loads(open('$OUT/b.json').read().strip().splitlines()[-1]); r=d['roofline']
print('$c $v', round(d['value']/1e6,1), 'Mevals/s', round(d['ms_per_step'],4), 'ms', {k:(round(v['ms_per_launch'],4),v['launches']) for k,v in r['per_kernel'].items()})"
done; done
