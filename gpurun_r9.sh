mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "perturbation or star or full_size or scaled" > gpurun_out/pytest9.log 2>&1; echo pytest=$? >> gpurun_out/pytest9.log
for kv in 0 7; do
for c in road rmat er; do
  SSSP_KVAR=$kv timeout 600 python tools/sweep.py --config $c --sources 4 --sets '[{}]' 2>&1 | sed "s/^/kv=$kv /" >> gpurun_out/sw9.log
done; done
timeout 600 python tools/sweep.py --config road --sources 4 --deltas 10,11,12,13 >> gpurun_out/sw9_roadstatic.log 2>&1
timeout 300 python tools/trace.py --config road --rows 40 > gpurun_out/trace9_road.log 2>&1
