set -x
mkdir -p gpurun_out
for c in road rmat er; do timeout 300 python tools/trace.py --config $c --rows 30 > gpurun_out/trace_$c.log 2>&1; done
timeout 600 python tools/sweep.py --config road --sources 6 --sets '[{}, {"delta_heuristic": 1}]' --deltas 11,12,13 > gpurun_out/sw_road.log 2>&1
timeout 600 python tools/sweep.py --config rmat --sources 4 --profile --sets '[{}]' --deltas 3 > gpurun_out/sw_rmat.log 2>&1
timeout 600 python tools/sweep.py --config er --sources 4 --profile --sets '[{}]' --deltas 15 > gpurun_out/sw_er.log 2>&1
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:adds_persistent -s 1 -c 1 \
      -o gpurun_out/r01_full_road python tools/sweep.py --config road --sources 1 --sets '[{"timeout_ms": 3600000}]' > gpurun_out/r01_full_road.log 2>&1
