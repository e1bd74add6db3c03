mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "perturbation or golden or scaled" > gpurun_out/pytest12.log 2>&1; echo pytest=$? >> gpurun_out/pytest12.log
for rep in 1 2; do
for ex in 0 1; do
  SSSP_EXP=$ex timeout 600 python tools/sweep.py --config road --sources 4 --sets '[{}]' --deltas 12 2>&1 | sed "s/^/exp=$ex /" >> gpurun_out/sw12.log
done; done
timeout 900 python bench.py --config batch --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/bench12_batch.log 2>&1
