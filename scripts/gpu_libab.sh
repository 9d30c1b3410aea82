#!/bin/bash
# A/B of two library builds on the resnet18 bench: variants/libbted_<name>.so vs the in-tree build.
# Usage: bash scripts/gpu_libab.sh <tag> <name> [reps] [config]
TAG=${1:-libab}; NAME=${2:-head}; REPS=${3:-3}; CFG=${4:-resnet18}
OUT=gpurun_out/$TAG; mkdir -p $OUT
LIB=paper_conf_date_sunbg021_b200/libbted.so
cp $LIB /tmp/libbted_new.so
for r in $(seq 1 $REPS); do
  for v in new $NAME; do
    if [ $v = new ]; then cp /tmp/libbted_new.so $LIB; else cp variants/libbted_$v.so $LIB; fi
    timeout 300 python bench.py --config $CFG --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/${v}_$r.json 2> $OUT/${v}_$r.err
  done
done
cp /tmp/libbted_new.so $LIB
for f in $OUT/*.json; do python -c "import json; d=json.load(open('$f')); print('$f', round(d['value'],1), round(d['ms_per_step'],3), round((d['roofline'].get('avg_launch_ms') or 0)*1e3,2), d['clocks']['sm_mhz'])" 2>&1 | tail -1; done | tee $OUT/summary.txt
