#!/bin/bash
# Iteration on the recomputing K.l pass: its tests, the parity tests of the implicit engine, bench, launch list.
TAG=${1:-rc}
OUT=gpurun_out/$TAG
mkdir -p $OUT
timeout 300 python -m pytest tests/test_gpu_recompute.py -m gpu -q -x -s > $OUT/rc.log 2>&1; echo "rc=$?" >> $OUT/rc.log
tail -3 $OUT/rc.log
grep -q "rc=0" $OUT/rc.log || exit 0
timeout 900 python -m pytest tests -m gpu -q -x -k "${2:-parity or k4 or fullsize}" > $OUT/pytest.log 2>&1; echo "rc=$?" >> $OUT/pytest.log
tail -3 $OUT/pytest.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $OUT/bench.json 2> $OUT/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_launches.log 2>&1
[ -n "$NCU_RC" ] && timeout 600 ncu --set full --clock-control none --import-source on -k regex:"rc_pass_kernel" -s 3 -c 1 \
    -o $OUT/prof_rc python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_rc.log 2>&1
true
