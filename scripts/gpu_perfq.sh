#!/bin/bash
# Quick perf iteration: implicit parity subset + bench lines (resnet18, vgg16, persistent).
OUT=gpurun_out/${1:-perfq}
mkdir -p $OUT
timeout 600 python -m pytest tests -m gpu -q -x -k "implicit or persistent or resnet18 or k4" > $OUT/pytest.log 2>&1; echo "rc=$?" >> $OUT/pytest.log
for cfg in resnet18 vgg16; do
  timeout 300 python bench.py --config $cfg --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/b_$cfg.json 2>/dev/null
  python -c "import json; j=json.load(open('$OUT/b_$cfg.json')); print('$cfg', round(j['value'],1), round(j['roofline']['avg_launch_ms']*1e3,2), 'us/step', j['clocks']['sm_mhz'])" >> $OUT/summary.txt 2>&1
done
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --persistent > $OUT/b_persist.json 2>/dev/null
python -c "import json; j=json.load(open('$OUT/b_persist.json')); print('persistent', round(j['value'],1), round(j['roofline']['avg_launch_ms']*1e3,2), 'us/step')" >> $OUT/summary.txt 2>&1
tail -3 $OUT/pytest.log >> $OUT/summary.txt
cat $OUT/summary.txt
