#!/bin/bash
# Implicit engine on one GPU: parity tests, bench line, ncu launch list + full captures.
OUT=gpurun_out/${1:-imp}
mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -k "implicit or k4 or subnormal" > $OUT/pytest_imp.log 2>&1; echo "rc=$?" >> $OUT/pytest_imp.log
timeout 600 python bench.py --steps 10 --warmup 3 --layout implicit --no-cpu-baseline > $OUT/bench_implicit.json 2> $OUT/bench_implicit.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --layout implicit > $OUT/ncu_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"tile_pass|ell_kernel|fin64" -s 30 -c 3 \
    -o $OUT/prof_imp python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --layout implicit > $OUT/ncu_imp.log 2>&1
