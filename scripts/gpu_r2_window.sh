#!/bin/bash
# Round 2: window-major path parity + timing + launch list.
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { cat $OUT/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_window.py -x -q > $OUT/pytest_window.log 2>&1; echo "window tests rc=$?"
tail -3 $OUT/pytest_window.log
B="python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-slowdown --no-per-config"
for wl in ${WLS:-12 13 14}; do
timeout 300 $B --replay-mode window --window-log2 $wl > $OUT/bench_cfg5_window_wl$wl.json 2> $OUT/bench_cfg5_window_wl$wl.err; echo "bench wl$wl rc=$?"
tail -2 $OUT/bench_cfg5_window_wl$wl.err
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file $OUT/launches_cfg5_window_wl$wl.csv $B --steps 1 --no-graph --replay-mode window --window-log2 $wl > $OUT/ncu_cfg5_window.log 2>&1; echo "ncu rc=$?"
done
