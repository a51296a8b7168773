#!/bin/bash
# ncu evidence for one round (run on the GPU box through gpurun, from the repo root):
#   tools/profile.sh <round> <config>
# 1. the launch list of the default bench command (gpu__time_duration.sum, --clock-control none)
# 2. one --set full capture of the two hot k_slots launches (forward map, reverse unmap) of a timed step
# Results land in gpurun_out/<round>/; summarise them here with tools/ncu_summary.py.
set -u
R=${1:-r01}
C=${2:-E}
mkdir -p gpurun_out/$R
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/$R/launches_$C.csv \
  python bench.py --config $C --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/$R/launches_${C}_stdout.txt 2>&1
# skip the 3 warm-up steps (2 hot launches each) and the setup launches; capture fwd + rev of one step
ncu --set full --clock-control none --import-source on -k regex:"k_fwd_fast|k_rev_fast" -s 6 -c 2 -o gpurun_out/$R/prof_$C -f \
  python bench.py --config $C --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/$R/full_${C}_stdout.txt 2>&1
ls -la gpurun_out/$R
