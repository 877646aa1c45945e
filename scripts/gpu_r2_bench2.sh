#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { cat $OUT/build.log; exit 1; }
( time timeout 1500 python bench.py ) > $OUT/bench_default.json 2> $OUT/bench_default.err
tail -c 1500 $OUT/bench_default.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file $OUT/launches_cfg5_default.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-slowdown \
  --no-per-config --no-graph > $OUT/ncu_cfg5.log 2>&1; echo "ncu rc=$?"
