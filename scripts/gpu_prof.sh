#!/bin/bash
# ncu evidence for the bench workload: the launch list (gpu__time_duration, cold-cache,
# serialised) and --set full captures of the top kernels.  Usage: bash scripts/gpu_prof.sh <tag> [config]
TAG=${1:-r2prof}
CFG=${2:-resnet18}
OUT=gpurun_out/$TAG
mkdir -p $OUT
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_$CFG.csv \
    python bench.py --config $CFG --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_launches_$CFG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"tile_pass|ell_kernel|fin64" -s 30 -c 3 \
    -o $OUT/prof_imp python bench.py --config $CFG --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_imp.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"gram_tc|prep_kernel|center_kernel" -s 3 -c 3 \
    -o $OUT/prof_gram python bench.py --config $CFG --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_gram.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"ted_cluster|ted_tiny" -s 3 -c 1 \
    -o $OUT/prof_merge python bench.py --config $CFG --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_merge.log 2>&1
ls -la $OUT
