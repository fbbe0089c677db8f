cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2n; mkdir -p $OUT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > $OUT/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_svr.py -x -q -k "test_svr_ragged_sizes_and_raw_mode and tcgen05 and 300" > $OUT/pytest1.log 2>&1; echo rc=$?; tail -25 $OUT/pytest1.log
timeout 900 python -m pytest tests/test_gpu_svr.py -x -q > $OUT/pytest.log 2>&1; echo rc=$?; tail -25 $OUT/pytest.log
