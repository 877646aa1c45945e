#!/bin/bash
# Round-2 ncu evidence: full capture of k_replay on config 2 (and 4), section capture on config 5.
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { cat $OUT/build.log; exit 1; }
B="python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-slowdown --no-per-config --no-graph"
for cfg in 2 4; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_replay -s 3 -c 1 \
  -o $OUT/r2_k_replay_cfg$cfg -f $B --config $cfg > $OUT/ncu_full_cfg$cfg.log 2>&1; echo "cfg$cfg rc=$?"
done
timeout 1500 ncu --section SpeedOfLight --section MemoryWorkloadAnalysis --section Occupancy --section WarpStateStats \
  --section LaunchStats --section SchedulerStats --clock-control none -k regex:k_replay -s 3 -c 1 \
  -o $OUT/r2_k_replay_cfg5 -f $B --config 5 > $OUT/ncu_sec_cfg5.log 2>&1; echo "cfg5 rc=$?"
tail -3 $OUT/ncu_sec_cfg5.log
