cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2b; mkdir -p $OUT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > $OUT/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q --durations=15 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -25 $OUT/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > $OUT/smoke.log 2>&1; tail -2 $OUT/smoke.log
timeout 600 python bench.py --steps 20 --warmup 5 > $OUT/bench_c3.json 2> $OUT/bench_c3.err; tail -c 2500 $OUT/bench_c3.json; tail -5 $OUT/bench_c3.err
for c in c1 c2 c5; do timeout 300 python bench.py --config $c --steps 20 --warmup 5 --no-cpu-baseline > $OUT/bench_$c.json 2> $OUT/bench_$c.err; tail -c 300 $OUT/bench_$c.json; done
for t in memcheck racecheck; do
  m=full; [ $t = racecheck ] && m=small
  SYNERGY_ALGO=1 timeout 600 compute-sanitizer --tool $t --print-limit 30 python scripts/sanitize_cases.py $m > $OUT/san_gen_$t.log 2>&1; echo $t rc=$?; tail -2 $OUT/san_gen_$t.log
done
timeout 600 compute-sanitizer --tool memcheck --print-limit 30 python scripts/sanitize_cases.py full > $OUT/san_tm_memcheck.log 2>&1; tail -2 $OUT/san_tm_memcheck.log
