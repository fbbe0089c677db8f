cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r3e; mkdir -p $OUT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > $OUT/build.log 2>&1
( time timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_streams_graphs.py tests/test_gpu_svr.py -m gpu -x -q -k "small or c1 or fuzz or capture or svr" ) > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log; tail -4 $OUT/pytest_gpu.log
bash scripts/ab_gpu.sh r3e "c1" "X=0" 2
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_tm_small -s 3 -c 1 -o $OUT/prof_small_c1 -f python bench.py --config c1 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_c1.log 2>&1
