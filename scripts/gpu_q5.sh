#!/bin/bash
# implicit engine: parity subset, split vs persistent bench lines, ablation, phase trace
OUT=gpurun_out/${1:-q5}; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x -k "implicit or persistent or launch or k4 or subnormal or resnet18 or identity or dup" > $OUT/pytest.log 2>&1; echo "rc=$?" >> $OUT/pytest.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --persistent > $OUT/bench_persistent.json 2> $OUT/bench_persistent.err
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/bench.json 2> $OUT/bench.err
timeout 300 python bench.py --config vgg16 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --persistent > $OUT/vgg_persistent.json 2> $OUT/vgg_p.err
timeout 300 python bench.py --config vgg16 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/vgg.json 2> $OUT/vgg.err
timeout 120 scripts/tp_ablate 16384 > $OUT/tp_ablate.txt 2>&1
timeout 300 python scripts/trace_loop.py 16384 $OUT/trace16k.txt > $OUT/trace.log 2>&1
