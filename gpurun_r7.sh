mkdir -p gpurun_out
for kv in 0 1; do
  for c in rmat er road; do
    d=$( [ $c = road ] && echo 12 || ([ $c = rmat ] && echo 3 || echo 15))
    SSSP_KVAR=$kv timeout 300 python tools/sweep.py --config $c --sources 4 --sets '[{}]' --deltas $d 2>&1 | sed "s/^/kv=$kv /" >> gpurun_out/ab7.log
  done
done
SSSP_KVAR=3 timeout 300 python tools/sweep.py --config rmat --sources 1 --deltas 3 > gpurun_out/kv3.log 2>&1
timeout 300 python tools/trace.py --config road --rows 40 > gpurun_out/trace7_road.log 2>&1
