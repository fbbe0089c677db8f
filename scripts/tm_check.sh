#!/bin/bash
# k_tm_walk: focused parity tests, then bench the given configs (env passes through)
OUT=gpurun_out/${1:-tmc}; mkdir -p $OUT
python -c "import paper_conf_sc_fandccfc23_b200.build as b; b.build()" > $OUT/build.log 2>&1 || { tail $OUT/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "${TESTK:-default or tm_ or routing or exact_sum or full_size}" > $OUT/pytest.log 2>&1; tail -2 $OUT/pytest.log
for c in ${CFGS:-c1 c2 c5 c3}; do
  timeout 300 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cpu-baseline --no-e2e > $OUT/bench_${c}.json 2> $OUT/bench_${c}.err
  python -c "import json;d=json.loads(open('$OUT/bench_${c}.json').read().strip().splitlines()[-1]);r=d['roofline'];print('$c', '%.4g'%d['value'], 'ms=%.4f'%d['ms_per_step'], {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})" 2>&1 | tail -1
done
