#!/bin/bash
# L2 policy sweep: BTED_L2_POLMODE x BTED_L2_KEEP_MB on resnet18 / vgg16 (implicit engine)
OUT=gpurun_out/${1:-l2sweep2}
mkdir -p $OUT
for pm in "0 0" "0 16" "1 0" "1 32" "1 64" "4 32" "4 64" "4 96" "4 126" "5 0"; do
  set -- $pm
  for cfg in resnet18 vgg16; do
    BTED_L2_POLMODE=$1 BTED_L2_KEEP_MB=$2 timeout 300 python bench.py --config $cfg --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/b.json 2>/dev/null
    python -c "import json,sys; j=json.load(open('$OUT/b.json')); print('$cfg mode=$1 keep=$2', round(j['value'],1), round(j['roofline']['avg_launch_ms']*1e3,2), 'us/step')" >> $OUT/summary.txt 2>&1
  done
done
cat $OUT/summary.txt
