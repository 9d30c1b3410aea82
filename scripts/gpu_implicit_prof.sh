#!/bin/bash
OUT=gpurun_out/${1:-imp}
mkdir -p $OUT
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --layout implicit > $OUT/ncu_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"tile_pass|ell_kernel|fin64" -s 30 -c 3 \
    -o $OUT/prof_imp python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --layout implicit > $OUT/ncu_imp.log 2>&1
