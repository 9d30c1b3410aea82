#!/bin/bash
# perfq + a warm ncu launch list of resnet18 (per-kernel durations)
OUT=gpurun_out/${1:-perfq2}
bash scripts/gpu_perfq.sh ${1:-perfq2}
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file $OUT/launches.csv \
    python bench.py --config resnet18 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python scripts/ncu_summary.py $OUT $OUT/sum > /dev/null 2>&1; head -8 $OUT/sum/ncu_summary.txt
