#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { cat $OUT/build.log; exit 1; }
for wl in 13 14; do
WL=$wl REPS=2 BLOCKS=1024 WORDS_LOG2=26 timeout 300 compute-sanitizer --tool memcheck --print-limit 3 python scripts/prof_window.py > $OUT/memcheck_wl$wl.log 2>&1
grep -v "Host Frame" $OUT/memcheck_wl$wl.log | tail -4
done
