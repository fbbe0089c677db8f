cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r3d; mkdir -p $OUT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > $OUT/build.log 2>&1
( time timeout 1500 python -m pytest tests -m gpu -x -q --durations=5 ) > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log; tail -4 $OUT/pytest_gpu.log
bash scripts/ab_gpu.sh r3d "c1 c2 c5" "X=0" 2
timeout 600 python bench.py > $OUT/bench_c3.json 2> $OUT/bench_c3.err; tail -c 300 $OUT/bench_c3.json
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_tm_finish -s 3 -c 1 -o $OUT/prof_finish_c2 -f python bench.py --config c2 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_c2.log 2>&1
(cd _ab/base && timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_tm_finish -s 3 -c 1 -o ../../$OUT/prof_finish_c2_base -f python bench.py --config c2 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > ../../$OUT/ncu_c2_base.log 2>&1)
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_tm_small -s 3 -c 1 -o $OUT/prof_small_c1 -f python bench.py --config c1 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_c1.log 2>&1
for t in memcheck racecheck; do
  m=full; [ $t = racecheck ] && m=small
  timeout 900 compute-sanitizer --tool $t --print-limit 30 python scripts/sanitize_cases.py $m > $OUT/san_$t.log 2>&1; echo $t rc=$?; tail -1 $OUT/san_$t.log
done
