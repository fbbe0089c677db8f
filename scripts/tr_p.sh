#!/bin/bash
# k_tr_walk chunk-size sweep on c2/c3 (bench only)
OUT=gpurun_out/${1:-trp}; mkdir -p $OUT
python -c "import paper_conf_sc_fandccfc23_b200.build as b; b.build()" > $OUT/build.log 2>&1
for c in c3 c2; do for p in ${PS:-512 1024 2048}; do
  SYNERGY_TR_P=$p timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/b_${c}_$p.json 2>$OUT/b_${c}_$p.err
  python -c "import json;d=json.loads(open('$OUT/b_${c}_$p.json').read().strip().splitlines()[-1]);r=d['roofline'];print('$c P=$p', 'ms=%.4f'%d['ms_per_step'], {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})" 2>&1 | tail -1
done; done
