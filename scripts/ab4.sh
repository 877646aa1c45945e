#!/bin/bash
# A/B of build/variants/*.so: bench timing per config + dynamic instruction count of k_replay (ncu).
OUT=gpurun_out; mkdir -p $OUT; rm -f $OUT/ab_summary.txt
for rep in $(seq ${REPS:-1}); do
for cfg in ${CFGS:-2 4}; do
for so in build/variants/*.so; do
  v=$(basename $so .so)
  HIRACE_LIB=$PWD/$so timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-slowdown --steps 50 --no-per-config --config $cfg > $OUT/ab_tmp.json 2>/dev/null
  inst=""
  if [ "$cfg" = "2" ]; then
    HIRACE_LIB=$PWD/$so timeout 300 ncu --metrics smsp__inst_executed.sum --clock-control none -k regex:k_replay -s 3 -c 1 --csv \
      python bench.py --no-cpu-baseline --no-e2e --no-slowdown --steps 2 --warmup 3 --config $cfg 2>/dev/null > $OUT/ab_ncu.csv
    inst=$(grep inst_executed $OUT/ab_ncu.csv | tail -1 | awk -F'","' '{print $NF}' | tr -d '",')
  fi
  python -c "import json; d=json.load(open('$OUT/ab_tmp.json')); print('cfg$cfg', '$v', round(d['roofline']['kernel_ms']*1000,1), 'us', round(d['roofline']['frac'],3), 'retries', d['check']['per_step']['cas_retries'], 'inst $inst')" >> $OUT/ab_summary.txt 2>&1
done; done; done
cat $OUT/ab_summary.txt
