cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2c; mkdir -p $OUT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > $OUT/build.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_c3.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_launch_bench.json 2>&1
tail -3 $OUT/launches_c3.csv
for c in c3 c2; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tm_walk -s 3 -c 1 \
  -o $OUT/prof_walk_$c -f python bench.py --config $c --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_full_$c.log 2>&1
tail -2 $OUT/ncu_full_$c.log
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tm_finish -s 3 -c 1 \
  -o $OUT/prof_finish_c2 -f python bench.py --config c2 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_full_fin_c2.log 2>&1
ls -la $OUT
