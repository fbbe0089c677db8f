#!/bin/bash
# L2 flush on/off A/B for the given configs (is the walk bound by cold model reads?)
OUT=gpurun_out/${1:-fab}; shift; mkdir -p $OUT
python -c "import paper_conf_sc_fandccfc23_b200.build as b; b.build()" > $OUT/build.log 2>&1
for c in ${@:-c2}; do for fl in 512 0; do
  timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --flush-mib $fl > $OUT/b_${c}_$fl.json 2>$OUT/b_${c}_$fl.err
  python -c "import json;d=json.loads(open('$OUT/b_${c}_$fl.json').read().strip().splitlines()[-1]);r=d['roofline'];print('$c flush=$fl', 'ms=%.4f'%d['ms_per_step'], {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})" 2>&1 | tail -1
done; done
