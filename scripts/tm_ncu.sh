#!/bin/bash
# ncu --set full (with source) of the tree-major kernels on the given configs
OUT=gpurun_out/${1:-tmn}; shift
mkdir -p $OUT
python -c "import paper_conf_sc_fandccfc23_b200.build as b; b.build()" > $OUT/build.log 2>&1
for c in ${@:-c2}; do
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_tm -s 4 -c 2 -o $OUT/tm_$c -f python bench.py --config $c --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_$c.log 2>&1; tail -1 $OUT/ncu_$c.log
done
