#!/bin/bash
# Round-2 final ncu evidence on the committed tree: full captures of k_replay (configs 2, 3, 4),
# section capture (config 5), launch list of the config-5 bench step, DRAM traffic per config.
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { cat $OUT/build.log; exit 1; }
B="python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-slowdown --no-per-config --no-graph"
for cfg in 2 3 4; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_replay -s 3 -c 1 \
  -o $OUT/r2b_k_replay_cfg$cfg -f $B --config $cfg > $OUT/ncu_full_cfg$cfg.log 2>&1; echo "cfg$cfg rc=$?"
done
timeout 1500 ncu --section SpeedOfLight --section MemoryWorkloadAnalysis --section Occupancy --section WarpStateStats \
  --section LaunchStats --section SchedulerStats --clock-control none -k regex:k_replay -s 3 -c 1 \
  -o $OUT/r2b_k_replay_cfg5 -f $B --config 5 > $OUT/ncu_sec_cfg5.log 2>&1; echo "cfg5 rc=$?"
timeout 1500 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 400 --csv \
  --log-file $OUT/r2b_launches_cfg5.csv python bench.py --steps 2 --warmup 3 --no-per-config --no-slowdown \
  --no-cpu-baseline --no-e2e --no-graph > $OUT/ncu_launches_cfg5.log 2>&1; echo "launches rc=$?"
for cfg in 2 3 4 6; do
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    -k regex:k_replay -s 3 -c 1 --csv --log-file $OUT/r2b_traffic_cfg$cfg.csv $B --config $cfg > $OUT/traffic_cfg$cfg.log 2>&1
done
ls -la $OUT | tail -20
