#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT; rm -f $OUT/ab_summary.txt
for so in build/variants/*.so; do
  v=$(basename $so .so)
  for h in "" "--no-hint"; do
    HIRACE_LIB=$PWD/$so timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-slowdown --steps 100 $h ${BENCH_ARGS} > $OUT/ab_tmp.json 2>/dev/null
    python -c "import json; d=json.load(open('$OUT/ab_tmp.json')); print('$v', '$h', round(d['roofline']['kernel_ms']*1000,1), 'us', round(d['ms_per_step']*1000,1), 'us/step', round(d['roofline']['frac'],3))" >> $OUT/ab_summary.txt 2>&1
  done
done
cat $OUT/ab_summary.txt
