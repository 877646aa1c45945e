#!/bin/bash
# smoke, masked-sync bench line (config 6) and an ncu capture of k_replay_masked
OUT=gpurun_out
mkdir -p $OUT
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke_m.log 2>&1; echo "smoke exit $?" >> $OUT/smoke_m.log
timeout 600 python bench.py --config 6 --steps 10 --warmup 3 --no-cpu-baseline --no-slowdown --no-per-config --no-e2e > $OUT/bench_cfg6.json 2> $OUT/bench_cfg6.err
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file $OUT/launches_cfg6.csv python bench.py --config 6 --steps 1 --warmup 1 --no-cpu-baseline --no-slowdown --no-per-config --no-e2e --no-graph > $OUT/ncu_cfg6.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_replay_masked -s 2 -c 1 \
    -o $OUT/prof_masked -f python bench.py --config 6 --steps 1 --warmup 2 --no-cpu-baseline --no-slowdown --no-per-config --no-e2e --no-graph > $OUT/ncu_masked_full.log 2>&1
echo done
