#!/bin/bash
# Quick GPU iteration: selected parity tests, bench line, warm launch list, read-bandwidth ceiling.
# Usage: bash scripts/gpu_quick.sh <tag> [pytest -k expr]
OUT=gpurun_out/${1:-quick}
K=${2:-"implicit or persistent or launch or k4 or subnormal or resnet18"}
mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x -k "$K" > $OUT/pytest.log 2>&1; echo "rc=$?" >> $OUT/pytest.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $OUT/bench.json 2> $OUT/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_launches.log 2>&1
[ -x scripts/read_bw ] && timeout 120 scripts/read_bw > $OUT/read_bw.txt 2>&1
