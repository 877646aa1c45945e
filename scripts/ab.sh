#!/bin/bash
# A/B timing of library variants in build/variants/*.so on the bench workload (no ncu).
OUT=gpurun_out; mkdir -p $OUT
for so in build/variants/*.so; do
  v=$(basename $so .so)
  HIRACE_LIB=$PWD/$so timeout 300 python bench.py --no-cpu-baseline --no-e2e --steps 100 ${BENCH_ARGS} > $OUT/ab_$v.json 2> $OUT/ab_$v.err
  python -c "import json; d=json.load(open('$OUT/ab_$v.json')); print('$v', round(d['roofline']['kernel_ms']*1000,1), 'us', round(d['roofline']['frac'],3), d['check']['per_step'])" >> $OUT/ab_summary.txt 2>&1
done
cat $OUT/ab_summary.txt
