#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
HIRACE_LIB=$PWD/build/variants/new.so timeout 900 python -m pytest tests/test_gpu_masked.py -x -q > $OUT/pytest_masked_new.log 2>&1; echo "rc=$?" >> $OUT/pytest_masked_new.log
rm -f $OUT/ab_masked2.txt
for rep in 1 2; do for v in old new; do
HIRACE_LIB=$PWD/build/variants/$v.so timeout 600 python bench.py --config 6 --steps 10 --warmup 3 --no-cpu-baseline --no-slowdown --no-per-config --no-e2e > $OUT/bench_cfg6_$v.json 2> /dev/null
python -c "import json; d=json.loads(open('$OUT/bench_cfg6_$v.json').read().strip().splitlines()[-1]); print('$v', d['ms_per_step'], d['roofline']['kernel_ms'])" >> $OUT/ab_masked2.txt
done; done
