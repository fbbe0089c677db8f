#!/bin/bash
bash scripts/gpu_round.sh r1p tests
OUT=gpurun_out/r1p_ab; mkdir -p $OUT
for c in c2 c3 c5 c4; do for pair in 0 1; do for kpc in 1 2 4; do
  if [ $c = c3 ] && [ $kpc != 1 ]; then continue; fi
  SYNERGY_PAIR=$pair SYNERGY_KPC=$kpc timeout 300 python bench.py --config $c --steps 5 --warmup 2 --no-cpu-baseline --no-e2e > $OUT/${c}_p${pair}_k$kpc.json 2>&1
  python -c "import json;d=json.load(open('$OUT/${c}_p${pair}_k$kpc.json'));print('$c pair=$pair kpc=$kpc', '%.3e'%d['value'], d['ms_per_step'])"
done; done; done
