#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_masked_inline.py -q -x > $OUT/pytest_mi2.log 2>&1; echo "rc=$?" >> $OUT/pytest_mi2.log
timeout 600 python -c "
import json, bench
print(json.dumps(bench.measure_slowdown(0), indent=1))" > $OUT/slowdown2.json 2> $OUT/slowdown2.err
