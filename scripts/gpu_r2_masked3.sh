#!/bin/bash
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { cat $OUT/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_masked.py -x -q > $OUT/pytest_masked.log 2>&1
echo "pytest exit $?" >> $OUT/pytest_masked.log
timeout 600 python bench.py --config 6 --steps 10 --warmup 3 --no-cpu-baseline --no-slowdown --no-per-config --no-e2e > $OUT/bench_cfg6.json 2> $OUT/bench_cfg6.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_replay_masked -s 2 -c 1 \
    -o $OUT/prof_masked -f python bench.py --config 6 --steps 1 --warmup 2 --no-cpu-baseline --no-slowdown --no-per-config --no-e2e --no-graph > $OUT/ncu_masked_full.log 2>&1
