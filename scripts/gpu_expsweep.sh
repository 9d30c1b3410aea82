#!/bin/bash
# A/B sweep of BTED_TP_EXP (bits 0-3 L2 prefetch tiles per CTA, 4 K-before-w, 5 early ell trigger)
OUT=gpurun_out/${1:-exps}
mkdir -p $OUT
for ex in 0 16 32 2 18 48 50 20 0; do
  for cfg in resnet18 vgg16; do
    BTED_TP_EXP=$ex timeout 300 python bench.py --config $cfg --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/b.json 2>/dev/null
    python -c "import json; j=json.load(open('$OUT/b.json')); print('$cfg exp=$ex', round(j['value'],1), round(j['roofline']['avg_launch_ms']*1e3,2), 'us/step', j['clocks']['sm_mhz'])" >> $OUT/summary.txt 2>&1
  done
done
cat $OUT/summary.txt
