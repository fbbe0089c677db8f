cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2i; mkdir -p $OUT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_streams_graphs.py -x -q > $OUT/pytest.log 2>&1; tail -2 $OUT/pytest.log
for c in c3 c2 c5 c1; do for v in "SYNERGY_TM_DYN=0" "SYNERGY_TM_DYN=1"; do
  env $v timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/b.json 2>/dev/null
  python -c "
import json,sys; d=json.loads(open('$OUT/b.json').read().strip().splitlines()[-1]); r=d['roofline']
print('$c $v', round(d['value']/1e6,1), 'Mevals/s', round(d['ms_per_step'],4), 'ms', {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})"
done; done
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_tm_walk -s 3 -c 1 -o $OUT/prof_walk_c3 -f python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu.log 2>&1; tail -1 $OUT/ncu.log
