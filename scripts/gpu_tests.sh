#!/bin/bash
# GPU session: the whole -m gpu suite (+ parity report), smoke.  Usage: bash scripts/gpu_tests.sh <tag> [pytest args]
TAG=${1:-r2}
shift
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/nvsmi.txt 2>&1
BTED_PARITY_REPORT=$OUT/parity_report.json timeout 2400 python -m pytest tests -m gpu -q -rA "$@" > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
tail -5 $OUT/pytest_gpu.log; tail -3 $OUT/smoke.log
