#!/bin/bash
# GPU session: bench lines.  Usage: bash scripts/gpu_bench.sh <tag> [configs...]
TAG=${1:-r2}
shift
OUT=gpurun_out/$TAG
mkdir -p $OUT
for cfg in "${@:-resnet18}"; do
  timeout 900 python bench.py --config $cfg --steps 10 --warmup 3 > $OUT/bench_$cfg.json 2> $OUT/bench_$cfg.err
  echo "$cfg rc=$?" >> $OUT/bench_rc.txt
done
cat $OUT/bench_rc.txt
