#!/bin/bash
# A/B of an environment switch on the implicit engine: parity subset + bench lines with and without it.
# Usage: bash scripts/gpu_ab.sh <tag> <ENV_VAR>
OUT=gpurun_out/${1:-ab}; V=${2:-BTED_FUSED_EB}
mkdir -p $OUT
env $V=1 timeout 600 python -m pytest tests -m gpu -q -x -k "implicit or persistent or resnet18 or k4 or toy or bted" > $OUT/pytest.log 2>&1; echo "rc=$?" >> $OUT/pytest.log
for rep in 1 2; do
for on in 0 1; do
  for cfg in resnet18 vgg16; do
    if [ $on = 1 ]; then E="env $V=1"; else E=""; fi
    $E timeout 300 python bench.py --config $cfg --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/b.json 2>/dev/null
    python -c "import json; j=json.load(open('$OUT/b.json')); print('$cfg $V=$on', round(j['value'],1), round(j['roofline']['avg_launch_ms']*1e3,2), 'us/step', j['clocks']['sm_mhz'])" >> $OUT/summary.txt 2>&1
  done
done
done
tail -2 $OUT/pytest.log >> $OUT/summary.txt
cat $OUT/summary.txt
