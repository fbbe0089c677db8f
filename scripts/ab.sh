#!/bin/bash
# A/B bench of the two sweep kernels on each config (device-resident, no CPU baseline / e2e)
OUT=gpurun_out/${1:-ab}
mkdir -p $OUT
for c in ${CFGS:-c2 c3 c5 c4 c1}; do
  for algo in ${ALGOS:-da ws direct}; do
    SYNERGY_ALGO=$algo timeout 600 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cpu-baseline --no-e2e > $OUT/$c.$algo.json 2> $OUT/$c.$algo.err
    python -c "
import json,sys
try:
  d=json.load(open('$OUT/$c.$algo.json')); r=d['roofline']
  print('$c $algo', 'evals/s %.3e'%d['value'], 'step_ms %.4f'%d['ms_per_step'], 'kern_ms %.4f'%r['kernel_ms'])
except Exception as e: print('$c $algo FAILED', e); print(open('$OUT/$c.$algo.err').read()[-1500:])
"
  done
done
