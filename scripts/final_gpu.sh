#!/bin/bash
# Round evidence on the current build (under gpurun): bench lines c1-c5 (+ SVR lines, reference
# arm), ncu launch list + full captures, the whole GPU suite with full-size c3 and c4 parity,
# smoke.  Usage: bash scripts/final_gpu.sh TAG
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-final}; mkdir -p $OUT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > $OUT/build.log 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv > $OUT/smi.txt 2>&1
# benches first (fresh box, cool GPU); default = c3 headline
timeout 900 python bench.py > $OUT/bench_c3.json 2> $OUT/bench_c3.err; tail -c 400 $OUT/bench_c3.json
for c in c1 c2 c4 c5; do
  timeout 900 python bench.py --config $c --steps 20 --warmup 5 > $OUT/bench_$c.json 2> $OUT/bench_$c.err; tail -c 200 $OUT/bench_$c.json
done
for c in c2 c3; do timeout 600 python bench.py --config $c --models svr --steps 10 --warmup 3 --no-cpu-baseline > $OUT/bench_${c}_svr.json 2> $OUT/bench_${c}_svr.err; done
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > $OUT/bench_ref_c3.json 2> $OUT/bench_ref_c3.err; tail -c 300 $OUT/bench_ref_c3.json
timeout 300 python __graft_entry__.py smoke > $OUT/smoke.log 2>&1; tail -n 2 $OUT/smoke.log
# launch list of the default bench, then ncu full captures
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_c3.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_launch_bench.json 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tm_walk -s 3 -c 1 -o $OUT/prof_walk_c3 -f python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_c3.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tm -s 6 -c 2 -o $OUT/prof_c2 -f python bench.py --config c2 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_svr_tc -s 2 -c 1 -o $OUT/prof_svr_tc_c3 -f python bench.py --config c3 --models svr --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_svr.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:k_tm_walk -s 3 -c 1 -o $OUT/prof_walk_c4 -f python bench.py --config c4 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_c4.log 2>&1
for r in prof_walk_c3 prof_c2 prof_svr_tc_c3 prof_walk_c4; do
  ncu -i $OUT/$r.ncu-rep --page raw --csv > $OUT/$r.raw.csv 2>/dev/null
done
ls $OUT
# tests: the whole GPU suite with full-size c3 and c4 (every row)
( time SYNERGY_FULL_PARITY=all timeout 3000 python -m pytest tests -m gpu -q --durations=8 ) > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log; tail -n 14 $OUT/pytest_gpu.log
cp gpurun_out/full_parity_c3.json gpurun_out/full_parity_c4.json $OUT/ 2>/dev/null
# compute-sanitizer is closed on the GPU pool (runs under it left GPUs needing a reset); the
# round's sanitizer logs are in profiles/r2/*sanitizer*
