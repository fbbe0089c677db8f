set -x
cd $GRAFT_REPO_ROOT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
nproc; free -g | head -2
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build()"
SYNERGY_FULL_PARITY=c4 timeout 1800 python -m pytest tests/test_gpu_fullsize.py -x -q -s > gpurun_out/r2a_fullsize.log 2>&1
echo fullsize rc=$?
for t in memcheck initcheck synccheck; do
  timeout 600 compute-sanitizer --tool $t --print-limit 30 python scripts/sanitize_cases.py full > gpurun_out/r2a_san_$t.log 2>&1; echo $t rc=$?
done
timeout 900 compute-sanitizer --tool racecheck --racecheck-report all --print-limit 30 python scripts/sanitize_cases.py small > gpurun_out/r2a_san_racecheck.log 2>&1; echo racecheck rc=$?
tail -3 gpurun_out/r2a_*.log
