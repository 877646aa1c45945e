#!/bin/bash
# Filter / granularity / inline round: build, targeted GPU tests, bench with slowdown.
TAG=${1:-q2}
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
timeout 900 python -m pytest tests/test_gpu_filter.py tests/test_gpu_granularity.py tests/test_gpu_inline.py tests/test_gpu_compact.py -x -q > $OUT/pytest_$TAG.log 2>&1
echo "pytest exit $?" >> $OUT/pytest_$TAG.log
timeout 600 python bench.py --no-cpu-baseline --no-e2e > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err
