OUT=gpurun_out/tpvar; mkdir -p $OUT
cp paper_conf_date_sunbg021_b200/libbted.so /tmp/libbted_orig.so
for rep in 1 2; do
for v in 0 1 4 5; do
  cp variants/libbted_v$v.so paper_conf_date_sunbg021_b200/libbted.so
  for cfg in oversized resnet18; do
    timeout 300 python bench.py --config $cfg --steps 6 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/${cfg}_v${v}_$rep.json 2> $OUT/${cfg}_v${v}_$rep.err
  done
done
done
cp /tmp/libbted_orig.so paper_conf_date_sunbg021_b200/libbted.so
for f in $OUT/*.json; do python -c "import json; d=json.load(open('$f')); print('$f', round(d['value'],1), round(d['ms_per_step'],3), round(d['roofline']['avg_launch_ms']*1e3,1), d['clocks']['sm_mhz'], d['clocks']['reasons'])" 2>&1 | tail -1; done | tee $OUT/summary.txt
