mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "perturbation or golden or scaled or star or full_size" > gpurun_out/pytest13.log 2>&1; echo pytest=$? >> gpurun_out/pytest13.log
for rep in 1 2; do
for ex in 0 2; do
for c in er rmat; do
  d=$( [ $c = rmat ] && echo 3 || echo 15)
  SSSP_EXP=$ex timeout 600 python tools/sweep.py --config $c --sources 3 --sets '[{}]' --deltas $d 2>&1 | sed "s/^/exp=$ex /" >> gpurun_out/sw13.log
done; done; done
