#!/bin/bash
# ncu evidence for the round's additions: compact vs 8-byte replay (config 3), the config-5
# launch list (report-buffer collect), and the config-3 k_replay full captures.
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_prof.log 2>&1
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-slowdown"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_replay -s 3 -c 1 \
  -o $OUT/prof_cfg3_compact -f $B --config 3 --compact > $OUT/ncu_cfg3c.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_replay -s 3 -c 1 \
  -o $OUT/prof_cfg3 -f $B --config 3 > $OUT/ncu_cfg3.log 2>&1
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_cfg5.csv \
  python bench.py --config 5 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-slowdown > $OUT/ncu_cfg5.log 2>&1
ls -la $OUT | tail -6
