#!/bin/bash
# Bench lines for the other BASELINE.json configurations on 1 GPU (profiles/).
OUT=gpurun_out/${1:-configs}
mkdir -p $OUT
timeout 900 python bench.py --config vgg16 --steps 3 --warmup 3 --scaling strong --no-cpu-baseline > $OUT/vgg16.json 2> $OUT/vgg16.err
timeout 900 python bench.py --config oversized --steps 3 --warmup 3 --no-cpu-baseline > $OUT/oversized.json 2> $OUT/oversized.err
timeout 900 python bench.py --config oversized --steps 3 --warmup 3 --no-cpu-baseline --layout packed > $OUT/oversized_packed.json 2> $OUT/oversized_packed.err
timeout 900 python bench.py --config paper --steps 10 --warmup 3 --no-cpu-baseline > $OUT/paper.json 2> $OUT/paper.err
timeout 600 python bench.py --config toy --steps 10 --warmup 3 --no-cpu-baseline > $OUT/toy.json 2> $OUT/toy.err
