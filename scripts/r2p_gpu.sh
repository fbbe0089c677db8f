cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2p; mkdir -p $OUT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_svr.py -x -q > $OUT/pytest.log 2>&1; echo rc=$?; tail -3 $OUT/pytest.log
for c in c2 c3; do for v in "SYNERGY_SVR_TC=1" "SYNERGY_SVR_TC=0"; do
  env $v timeout 600 python bench.py --config $c --models svr --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/svr_${c}_$v.json 2>$OUT/err.txt
  python -c "
import json,sys; d=json.loads(open('$OUT/svr_${c}_$v.json').read().strip().splitlines()[-1]); r=d['roofline']
print('$c $v', round(d['value']/1e6,1), 'Mevals/s', round(d['ms_per_step'],4), 'ms', r['kernel'], round(r['frac'],3), r.get('svr_contraction',{}).get('frac'), {k:(round(v['ms_per_launch'],4),v['launches']) for k,v in r['per_kernel'].items()})"
done; done
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_svr_tc -s 2 -c 1 -o $OUT/prof_svr_tc_c3 -f python bench.py --config c3 --models svr --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu.log 2>&1; tail -1 $OUT/ncu.log
