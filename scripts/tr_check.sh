#!/bin/bash
# k_tr_walk vs k_tm_walk: focused parity tests, then bench c2/c3 in both modes.
OUT=gpurun_out/${1:-trc}; mkdir -p $OUT
python -c "import paper_conf_sc_fandccfc23_b200.build as b; b.build()" > $OUT/build.log 2>&1 || { tail $OUT/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "default or tr_ or routing or exact_sum or full_size" > $OUT/pytest.log 2>&1; tail -3 $OUT/pytest.log
for c in ${CFGS:-c2 c3}; do
  for mode in tr tm; do
    SYNERGY_TM_MODE=$mode timeout 300 python bench.py --config $c --steps ${STEPS:-10} --warmup 3 --no-cpu-baseline --no-e2e > $OUT/bench_${c}_$mode.json 2> $OUT/bench_${c}_$mode.err
    python -c "import json;d=json.loads(open('$OUT/bench_${c}_$mode.json').read().strip().splitlines()[-1]);r=d['roofline'];print('$c $mode', '%.4g'%d['value'], 'ms=%.4f'%d['ms_per_step'], {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})" 2>&1 | tail -1
  done
done
