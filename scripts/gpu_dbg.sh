#!/bin/bash
for wl in 12 13 14; do for hv in "" 100000000; do
echo "== wl $wl heavy_force '$hv'"
HIRACE_WIN_HEAVY=$hv HIRACE_WIN_VALIDATE=1 WL=$wl REPS=1 timeout 120 python scripts/prof_window.py 2>&1 | tail -2
done; done
