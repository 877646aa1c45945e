#!/bin/bash
# Fast iteration: parity subset, bench (no CPU baseline), ncu full capture of k_replay.
TAG=${1:-q}
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "not full" > $OUT/pytest_gpu_$TAG.log 2>&1
echo "pytest exit $?" >> $OUT/pytest_gpu_$TAG.log
timeout 600 python bench.py --no-cpu-baseline ${BENCH_ARGS} > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_replay -s 3 -c 1 \
    -o $OUT/prof_replay_$TAG -f python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline ${BENCH_ARGS} > $OUT/ncu_full_$TAG.log 2>&1
