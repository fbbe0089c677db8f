#!/bin/bash
# bench one config under several environment settings: tm_env.sh TAG CFG "ENV1" "ENV2" ...
OUT=gpurun_out/$1; C=$2; shift 2; mkdir -p $OUT
python -c "import paper_conf_sc_fandccfc23_b200.build as b; b.build()" > $OUT/build.log 2>&1
i=0
for e in "$@"; do
  i=$((i+1))
  env $e timeout 300 python bench.py --config $C --steps ${STEPS:-20} --warmup 3 --no-cpu-baseline --no-e2e > $OUT/b_$i.json 2>$OUT/b_$i.err
  python -c "import json;d=json.loads(open('$OUT/b_$i.json').read().strip().splitlines()[-1]);r=d['roofline'];print('$C [$e]', 'ms=%.4f'%d['ms_per_step'], {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})" 2>&1 | tail -1
done
