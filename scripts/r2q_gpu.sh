cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2q; mkdir -p $OUT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > $OUT/build.log 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv > $OUT/smi.txt 2>&1
( time timeout 1500 python -m pytest tests -m gpu -q --durations=10 ) > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log; tail -16 $OUT/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > $OUT/smoke.log 2>&1; tail -2 $OUT/smoke.log
for t in memcheck racecheck synccheck initcheck; do
  m=full; [ $t = racecheck ] && m=small
  timeout 900 compute-sanitizer --tool $t --print-limit 30 python scripts/sanitize_cases.py $m > $OUT/san_$t.log 2>&1; echo $t rc=$?; tail -1 $OUT/san_$t.log
done
