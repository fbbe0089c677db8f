#!/bin/bash
# Tree-major path experiments: knob sweep on c2 (+flush off), ncu source capture of k_tm_walk.
OUT=gpurun_out/${1:-tmx}
mkdir -p $OUT
python -c "import paper_conf_sc_fandccfc23_b200.build as b; b.build()" > $OUT/build.log 2>&1
run() {  # name, env..., -- bench args
  local name=$1; shift
  env "$@" timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e $BARGS > $OUT/$name.json 2> $OUT/$name.err
  python -c "
import json
try:
  d=json.load(open('$OUT/$name.json')); print('$name', '%.3e'%d['value'], round(d['ms_per_step'],4), {k:round(v['ms_per_launch'],4) for k,v in d['roofline']['per_kernel'].items()})
except Exception as e: print('$name FAIL', e, open('$OUT/$name.err').read()[-1500:])
"
}
for c in c2 c1; do
  BARGS="--config $c" run ${c}_base X=1
  BARGS="--config $c --flush-mib 0" run ${c}_noflush X=1
  BARGS="--config $c" run ${c}_da SYNERGY_ALGO=da
  BARGS="--config $c --flush-mib 0" run ${c}_da_noflush SYNERGY_ALGO=da
done
BARGS="--config c2" run c2_ctas148 SYNERGY_TM_CTAS=148
BARGS="--config c2" run c2_ctas592 SYNERGY_TM_CTAS=592
BARGS="--config c2" run c2_kb64 SYNERGY_TM_KB=64
BARGS="--config c2" run c2_kb128 SYNERGY_TM_KB=128
BARGS="--config c3" run c3_base X=1
BARGS="--config c3" run c3_kb64 SYNERGY_TM_KB=64
for c in c2 c1; do
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_tm -s 4 -c 2 -o $OUT/tm_$c -f python bench.py --config $c --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_$c.log 2>&1; tail -1 $OUT/ncu_$c.log
done
