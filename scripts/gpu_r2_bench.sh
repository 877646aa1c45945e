#!/bin/bash
# Round 2: default bench (config 5 + per_config) and per-config DRAM traffic of k_replay.
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { cat $OUT/build.log; exit 1; }
( time timeout 1200 python bench.py ) > $OUT/bench_default.json 2> $OUT/bench_default.err
tail -c 3000 $OUT/bench_default.err
B="python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-slowdown --no-per-config --no-graph"
for cfg in 2 3 4 5; do
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    -k regex:k_replay -s 3 -c 1 --csv --log-file $OUT/traffic_cfg$cfg.csv $B --config $cfg > $OUT/traffic_cfg$cfg.log 2>&1
done
ls -la $OUT | tail -12
