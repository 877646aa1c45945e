#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { cat $OUT/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_masked_inline.py tests/test_gpu_inline.py tests/test_gpu_masked.py -q -x > $OUT/pytest_mi.log 2>&1; echo "rc=$?" >> $OUT/pytest_mi.log
timeout 600 python -c "
import json, bench
print(json.dumps(bench.measure_slowdown(0), indent=1))" > $OUT/slowdown.json 2> $OUT/slowdown.err
