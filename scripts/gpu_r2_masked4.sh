#!/bin/bash
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { cat $OUT/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_masked.py -x -q > $OUT/pytest_masked.log 2>&1
echo "pytest exit $?" >> $OUT/pytest_masked.log
rm -f $OUT/ab_masked.txt
for rep in 1 2; do for v in m3 m4; do
HIRACE_LIB=$PWD/build/variants/$v.so timeout 600 python bench.py --config 6 --steps 10 --warmup 3 --no-cpu-baseline --no-slowdown --no-per-config --no-e2e > $OUT/bench_cfg6_$v.json 2> $OUT/bench_cfg6.err
python -c "import json; d=json.loads(open('$OUT/bench_cfg6_$v.json').read().strip().splitlines()[-1]); print('$v', d['ms_per_step'], d['roofline']['kernel_ms'])" >> $OUT/ab_masked.txt
done; done
