#!/bin/bash
# A/B of library settings on the resnet18 bench: bash scripts/gpu_ab.sh <tag> "<ENV=VAL> ..." [reps] [bench args]
# (each setting's env assignment applies to one bench run; settings alternate, reps times)
TAG=${1:-ab}
SETS=${2:-"X=0"}
REPS=${3:-2}
ARGS=${4:-}
OUT=gpurun_out/$TAG
mkdir -p $OUT
for r in $(seq 1 $REPS); do
  for s in $SETS; do
    env $s timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e $ARGS > $OUT/bench_${s}_$r.json 2> $OUT/bench_${s}_$r.err
  done
done
for f in $OUT/bench_*.json; do
  python -c "import json; d=json.load(open('$f')); print('$f', round(d['value']), round(d['ms_per_step'],3), round(d['roofline']['avg_launch_ms']*1e3,1), d['clocks']['sm_mhz'])" 2>&1 | tail -1
done | tee $OUT/summary.txt
