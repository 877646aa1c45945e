#!/bin/bash
# A/B of build/variants/*.so on configs 2 and 4 (replay kernel + fused collect, per step)
OUT=gpurun_out; mkdir -p $OUT; rm -f $OUT/ab_summary.txt
for cfg in ${CFGS:-2 4}; do
for so in build/variants/*.so; do
  v=$(basename $so .so)
  HIRACE_LIB=$PWD/$so timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-slowdown --steps 50 --config $cfg > $OUT/ab_tmp.json 2>/dev/null
  python -c "import json; d=json.load(open('$OUT/ab_tmp.json')); print('cfg$cfg', '$v', round(d['roofline']['kernel_ms']*1000,1), 'us', round(d['roofline']['frac'],3), 'retries', d['check']['per_step']['cas_retries'])" >> $OUT/ab_summary.txt 2>&1
done; done
cat $OUT/ab_summary.txt
