#!/bin/bash
# Hybrid K.l pass (csrc/hy_pass.cuh) sweep: the streaming pass on an SM subset
# (scripts/sm_subset_probe.cu), then the resnet18 bench for BTED_HYBRID = R:frac settings.
# Usage: bash scripts/gpu_hybrid_sweep.sh <tag> "<R:frac> ..."
TAG=${1:-hy}
SETS=${2:-"24:0.09 32:0.12 40:0.155 48:0.19"}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/sm_subset_probe scripts/sm_subset_probe.cu \
  && timeout 120 /tmp/sm_subset_probe > $OUT/sm_subset.txt 2>&1
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/bench_off.json 2> $OUT/bench_off.err
for s in $SETS; do
  BTED_HYBRID=$s timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/bench_$s.json 2> $OUT/bench_$s.err
done
for f in $OUT/bench_*.json; do
  python -c "import json,sys; d=json.load(open('$f')); print('$f', round(d['value']), round(d['ms_per_step'],3), round(d['roofline']['avg_launch_ms']*1e3,1), d['clocks']['sm_mhz'])" 2>&1 | tail -1
done | tee $OUT/summary.txt
