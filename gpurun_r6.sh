mkdir -p gpurun_out
for kv in 0 1 2 3 4 5 6; do
  for c in rmat er road; do
    d=$( [ $c = road ] && echo 12 || ([ $c = rmat ] && echo 3 || echo 15))
    SSSP_KVAR=$kv timeout 300 python tools/sweep.py --config $c --sources 3 --deltas $d | sed "s/^/kv=$kv /" >> gpurun_out/ab6.log 2>&1
  done
done
