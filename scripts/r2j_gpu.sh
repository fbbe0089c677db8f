cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2j; mkdir -p $OUT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > $OUT/build.log 2>&1
for v in "SYNERGY_TM_SLAB=0" "SYNERGY_TM_SLAB=10240" "SYNERGY_TM_SLAB=7680" "SYNERGY_TM_SLAB=5120" "SYNERGY_TM_KB=128" "SYNERGY_TM_KB=128 SYNERGY_TM_SLAB=7680"; do
  env $v timeout 300 python bench.py --config c3 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/b.json 2>/dev/null
  python -c "
import json,sys; d=json.loads(open('$OUT/b.json').read().strip().splitlines()[-1]); r=d['roofline']
print('c3 $v', round(d['value']/1e6,1), 'Mevals/s', round(d['ms_per_step'],4), 'ms', {k:(round(v['ms_per_launch'],4),v['launches']) for k,v in r['per_kernel'].items()})"
done
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_tm -s 6 -c 2 -o $OUT/prof_c2 -f python bench.py --config c2 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu.log 2>&1; tail -1 $OUT/ncu.log
