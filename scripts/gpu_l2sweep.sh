#!/bin/bash
# Sweep of the L2 carry-over between K.l passes (BTED_L2_KEEP_MB) on the bench workloads.
OUT=gpurun_out/${1:-l2sweep}
mkdir -p $OUT
timeout 600 python -m pytest tests -m gpu -q -x -k "implicit or persistent or resnet18" > $OUT/pytest.log 2>&1; echo "rc=$?" >> $OUT/pytest.log
for mb in 0 32 48 64 80 96 112; do
  for cfg in resnet18 vgg16; do
    BTED_L2_KEEP_MB=$mb timeout 300 python bench.py --config $cfg --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/b_${cfg}_$mb.json 2>/dev/null
    python -c "import json,sys; j=json.load(open('$OUT/b_${cfg}_$mb.json')); print('$cfg', $mb, round(j['value'],1), round(j['roofline']['avg_launch_ms']*1e3,2), 'us/step')" >> $OUT/summary.txt 2>&1
  done
done
BTED_L2_KEEP_MB=64 timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --persistent > $OUT/b_persist_64.json 2>/dev/null
BTED_L2_KEEP_MB=0 timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --persistent > $OUT/b_persist_0.json 2>/dev/null
cat $OUT/summary.txt
