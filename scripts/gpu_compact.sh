#!/bin/bash
# Compact-record round: build, GPU tests (compact + full parity), bench 8-byte vs compact.
TAG=${1:-c}
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
timeout 600 python -m pytest tests/test_gpu_compact.py -x -q > $OUT/pytest_compact_$TAG.log 2>&1
echo "pytest exit $?" >> $OUT/pytest_compact_$TAG.log
timeout 900 python -m pytest tests -m gpu -x -q -k "not full and not compact" > $OUT/pytest_gpu_$TAG.log 2>&1
echo "pytest exit $?" >> $OUT/pytest_gpu_$TAG.log
for cfg in 2 3 4; do
  for mode in "" "--compact"; do
    name=cfg${cfg}${mode:+_compact}
    timeout 600 python bench.py --config $cfg $mode --no-cpu-baseline --no-slowdown --no-e2e --steps 50 > $OUT/bench_${name}_$TAG.json 2> $OUT/bench_${name}_$TAG.err
  done
done
timeout 600 python bench.py --config 3 --variant clean --no-cpu-baseline --no-slowdown --no-e2e --steps 30 > $OUT/bench_cfg3clean_$TAG.json 2>&1
timeout 600 python bench.py --config 3 --variant clean --compact --no-cpu-baseline --no-slowdown --no-e2e --steps 30 > $OUT/bench_cfg3clean_compact_$TAG.json 2>&1
ls -la $OUT | tail -30
