#!/bin/bash
# One GPU session: tests, smoke, bench (all three engines), ncu launch list + full captures.
# Usage (from the repo root, under gpurun): bash scripts/gpu_check.sh [tag] [pytest-args]
TAG=${1:-r1}
PYARGS=${2:-}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/nvsmi.txt 2>&1
BTED_PARITY_REPORT=$OUT/parity_report.json timeout 1200 python -m pytest tests -m gpu -q $PYARGS > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
timeout 120 python scripts/h2d_probe.py > $OUT/h2d.txt 2>&1
timeout 300 python __graft_entry__.py smoke > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
timeout 900 python bench.py --steps 10 --warmup 3 > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?" >> $OUT/bench.err
timeout 900 python bench.py --steps 10 --warmup 3 --layout dense --no-cpu-baseline > $OUT/bench_dense.json 2> $OUT/bench_dense.err
timeout 900 python bench.py --steps 10 --warmup 3 --layout packed --no-cpu-baseline > $OUT/bench_packed.json 2> $OUT/bench_packed.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"tile_pass|ell_kernel|fin64" -s 30 -c 3 \
    -o $OUT/prof_imp python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_imp.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"deflate_packed|finalize_packed" -s 16 -c 2 \
    -o $OUT/prof_k2p python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --layout packed > $OUT/ncu_k2p.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"gram_tile|gram_packed" -s 2 -c 1 \
    -o $OUT/prof_k1p python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_k1p.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:deflate_rescore -s 8 -c 1 \
    -o $OUT/prof_k2 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --layout dense > $OUT/ncu_k2.log 2>&1
ls -la $OUT
