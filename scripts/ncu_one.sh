#!/bin/bash
# ncu --set full (with source) of one kernel on given configs: ncu_one.sh TAG KERNEL_REGEX CFG... (env passes through)
OUT=gpurun_out/$1; K=$2; shift 2
mkdir -p $OUT
python -c "import paper_conf_sc_fandccfc23_b200.build as b; b.build()" > $OUT/build.log 2>&1
for c in ${@:-c2}; do
timeout 900 ncu --set full --import-source on --clock-control none -k regex:$K -s 2 -c 1 -o $OUT/${K}_$c -f python bench.py --config $c --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_$c.log 2>&1; tail -1 $OUT/ncu_$c.log
done
