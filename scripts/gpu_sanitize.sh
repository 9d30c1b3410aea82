#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over scripts/sanitize_cases.py.
TAG=${1:-r2san}
OUT=gpurun_out/$TAG
mkdir -p $OUT
CASES="${CASES:-toy tiny64 tiny33 tinybatches cluster500 cluster940 implicit4096 persistent4096 packed4096 packedtma4096 dense4096 k4full2048 recompute4096 recompute_guard tileshard3 rowbands2 bands_literal2 batches}"
for tool in memcheck racecheck synccheck; do
  for c in $CASES; do
    timeout 600 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 \
      python scripts/sanitize_cases.py $c > $OUT/${tool}_$c.log 2>&1
    echo "$tool $c rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' $OUT/${tool}_$c.log | tail -1)" >> $OUT/summary.txt
  done
done
cat $OUT/summary.txt
