#!/bin/bash
# Cluster-level replay on the GPU: parity tests, rate, launch list and one ncu capture.
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_cl.log 2>&1
timeout 600 python -m pytest tests/test_gpu_cluster.py -x -q > $OUT/pytest_cluster.log 2>&1; echo "exit $?" >> $OUT/pytest_cluster.log
timeout 300 python scripts/bench_cluster.py > $OUT/bench_cluster.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_cluster_replay -s 3 -c 1 \
  -o $OUT/prof_cluster -f python scripts/bench_cluster.py > $OUT/ncu_cluster.log 2>&1
ls -la $OUT | tail -8
