#!/bin/bash
# ncu evidence for one round (run on the GPU box from the repo root):
#  1. launch list of the bench command (per-launch device time, cold cache, serialised)
#  2. one --set full capture of the persistent kernel per config
set -x
R=${1:-r01}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${R}_launches_road.csv \
    python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline > gpurun_out/${R}_launches_road.log 2>&1
for c in road rmat er; do
  ncu --set full --import-source on --clock-control none -k regex:adds_persistent -s 1 -c 1 \
      -o gpurun_out/${R}_full_$c python tools/sweep.py --config $c --sources 1 --sets "[{}]" \
      > gpurun_out/${R}_full_$c.log 2>&1
done
