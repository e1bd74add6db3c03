#!/bin/bash
# ncu evidence for one round (run on the GPU box from the repo root):
#  1. launch list of the default bench command (per-launch device time, cold cache, serialised)
#  2. one --set full capture of the persistent kernel per config, in the launch shape the bench
#     times (singles: the default options of configs 2-4; batch: config 5 with 4 sources in flight)
set -x
R=${1:-r02}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${R}_launches.csv \
    python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline --single-steps 1 --single-warmup 1 \
    > gpurun_out/${R}_launches.log 2>&1
for c in road rmat er; do
  ncu --set full --import-source on --clock-control none -k regex:adds_persistent -s 1 -c 1 \
      -o gpurun_out/${R}_full_$c python tools/sweep.py --config $c --sources 1 --sets "[{}]" \
      > gpurun_out/${R}_full_$c.log 2>&1
done
ncu --set full --import-source on --clock-control none -k regex:adds_persistent -s 8 -c 1 \
    -o gpurun_out/${R}_full_batch python tools/batch_sweep.py --config batch --k 8 --conc 4 --reps 1 \
    > gpurun_out/${R}_full_batch.log 2>&1
