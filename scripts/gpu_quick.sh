#!/bin/bash
# Quick iteration: selected GPU tests, the bench line, the launch list.  Usage: bash scripts/gpu_quick.sh <tag> [-k expr]
TAG=${1:-quick}
K=${2:-"tensor_core or gram or identity or k4"}
OUT=gpurun_out/$TAG
mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x -k "$K" -s > $OUT/pytest.log 2>&1; echo "rc=$?" >> $OUT/pytest.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $OUT/bench.json 2> $OUT/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_launches.log 2>&1
tail -3 $OUT/pytest.log
[ -n "$NCU_GRAM" ] && timeout 600 ncu --set full --clock-control none --import-source on -k regex:"gram_tc_kernel" -s 1 -c 1 \
    -o $OUT/prof_gram python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_gram.log 2>&1
true
