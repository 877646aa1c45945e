#!/bin/bash
# Share-bias A/B (HIRACE_SLOT_BIAS): parity at one bias, then kernel time per bias and config.
OUT=gpurun_out; mkdir -p $OUT; rm -f $OUT/ab_bias.txt
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_bias.log 2>&1
HIRACE_SLOT_BIAS=0.15 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "not full and not cfg5" > $OUT/pytest_bias.log 2>&1
echo "pytest exit $?" >> $OUT/pytest_bias.log
for cfg in 2 4 3; do
  for b in 0 0.05 0.1 0.15 0.2 0.3; do
    HIRACE_SLOT_BIAS=$b timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-slowdown --steps 50 --config $cfg > $OUT/ab_tmp.json 2>/dev/null
    python -c "import json; d=json.load(open('$OUT/ab_tmp.json')); print('cfg$cfg', 'bias $b', round(d['roofline']['kernel_ms']*1000,1), 'us', round(d['roofline']['frac'],3), 'step', round(d['ms_per_step']*1000,1), 'retries', d['check']['per_step']['cas_retries'])" >> $OUT/ab_bias.txt 2>&1
  done
done
cat $OUT/ab_bias.txt
