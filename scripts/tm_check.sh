#!/bin/bash
# Tree-major path check: parity (default + tm variants), then c2/c3 benches against k_sweep_da.
OUT=gpurun_out/${1:-tm}
mkdir -p $OUT
python -c "import paper_conf_sc_fandccfc23_b200.build as b; b.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "default or tm_" > $OUT/pytest_tm.log 2>&1; echo "rc=$?" >> $OUT/pytest_tm.log
tail -5 $OUT/pytest_tm.log
for c in c2 c3 c5 c1; do
  timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/tm_$c.json 2> $OUT/tm_$c.err
  python -c "
import json
try:
  d=json.load(open('$OUT/tm_$c.json')); print('$c tm', '%.3e'%d['value'], d['ms_per_step'], {k:round(v['ms_per_launch'],4) for k,v in d['roofline']['per_kernel'].items()})
except Exception as e: print('$c FAIL', e, open('$OUT/tm_$c.err').read()[-2000:])
"
done
