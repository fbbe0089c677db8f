#!/bin/bash
# One GPU session: parity tests, benches, ncu launch list + full capture of the sweep kernel.
# Usage (under gpurun): bash scripts/gpu_round.sh [tag] [stages...]
#   stages: tests bench ncu full (default: all)
TAG=${1:-r1}
shift
STAGES=${@:-tests bench ncu full}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import paper_conf_sc_fandccfc23_b200.build as b; b.build()" > $OUT/build.log 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv > $OUT/smi.txt 2>&1
for s in $STAGES; do
  case $s in
    tests)
      timeout 900 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
      tail -3 $OUT/pytest_gpu.log ;;
    smoke)
      timeout 300 python __graft_entry__.py smoke > $OUT/smoke.log 2>&1; tail -2 $OUT/smoke.log ;;
    bench)
      timeout 600 python bench.py > $OUT/bench_c2.json 2> $OUT/bench_c2.err; tail -c 3000 $OUT/bench_c2.json
      for c in c1 c3 c4 c5; do
        timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > $OUT/bench_$c.json 2> $OUT/bench_$c.err
        tail -c 400 $OUT/bench_$c.json
      done ;;
    ref)
      timeout 600 python bench.py --impl reference --steps 5 --warmup 1 > $OUT/bench_ref.json 2> $OUT/bench_ref.err; tail -c 600 $OUT/bench_ref.json ;;
    ncu)
      timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_c2.csv \
        python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_launch_bench.json 2>&1
      tail -5 $OUT/launches_c2.csv ;;
    full)
      for c in ${NCU_CFGS:-c2}; do
        timeout 1200 ncu --set full --clock-control none --import-source on -k regex:${NCU_K:-k_tm_walk} -s 3 -c 1 \
          -o $OUT/prof_$c -f python bench.py --config $c --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $OUT/ncu_full_$c.log 2>&1
        tail -3 $OUT/ncu_full_$c.log
      done ;;
  esac
done
ls -la $OUT
