cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2d; mkdir -p $OUT
python -c "import tools; tools.build()" > $OUT/build.log 2>&1
python scripts/peaks_probe.py > $OUT/peaks_probe.json 2>&1; cat $OUT/peaks_probe.json
timeout 600 ncu --set full --clock-control none -k regex:k_scatter -c 6 -o $OUT/prof_peaks -f python scripts/peaks_probe.py > $OUT/ncu_peaks.log 2>&1; tail -2 $OUT/ncu_peaks.log
