#!/bin/bash
# Bench lines for the other BASELINE.json configurations on 1 GPU (profiles/).
OUT=gpurun_out/${1:-configs}
mkdir -p $OUT
timeout 900 python bench.py --config vgg16 --steps 3 --warmup 3 --scaling strong --no-cpu-baseline > $OUT/vgg16.json 2> $OUT/vgg16.err
timeout 1200 python bench.py --config oversized --steps 3 --warmup 3 > $OUT/oversized.json 2> $OUT/oversized.err
timeout 900 python bench.py --config oversized --steps 3 --warmup 3 --no-cpu-baseline --layout packed > $OUT/oversized_packed.json 2> $OUT/oversized_packed.err
timeout 900 python bench.py --config paper --steps 10 --warmup 3 --no-cpu-baseline > $OUT/paper.json 2> $OUT/paper.err
timeout 600 python bench.py --config toy --steps 10 --warmup 3 --no-cpu-baseline > $OUT/toy.json 2> $OUT/toy.err
timeout 1200 python bench.py --config wholemodel --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/wholemodel.json 2> $OUT/wholemodel.err
timeout 900 python bench.py --config large --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/large.json 2> $OUT/large.err
timeout 600 python bench.py --config resnet18 --steps 10 --warmup 3 --layout packed --no-cpu-baseline > $OUT/resnet18_packed.json 2> $OUT/resnet18_packed.err
timeout 600 python bench.py --config resnet18 --steps 20 --warmup 5 > $OUT/resnet18.json 2> $OUT/resnet18.err
timeout 900 python bench.py --impl reference --config resnet18 --steps 3 --warmup 3 > $OUT/reference_resnet18.json 2> $OUT/reference_resnet18.err
for f in $OUT/*.json; do python -c "
import json,sys
try:
    j=json.load(open('$f')); r=j.get('roofline') or {}
    print('$f'.split('/')[-1], round(j['value'],1), j['unit'], 'ms/step', round(j['ms_per_step'],3), 'achieved', r.get('achieved'), 'frac', r.get('frac'), 'clk', (j.get('clocks') or {}).get('sm_mhz'))
except Exception as e: print('$f', 'ERR', e)
"; done > $OUT/summary.txt
cat $OUT/summary.txt
