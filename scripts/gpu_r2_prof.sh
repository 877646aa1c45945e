#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { cat $OUT/build.log; exit 1; }
WL=${WL:-13} timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_w_light|k_w_scatter|k_w_heavy" -s 4 -c 4 \
  -o $OUT/prof_window -f python scripts/prof_window.py > $OUT/ncu_prof_window.log 2>&1; echo "ncu rc=$?"
tail -3 $OUT/ncu_prof_window.log
