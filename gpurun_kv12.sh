mkdir -p gpurun_out
for i in 1 2 3 4; do
  for kv in 0 2 6 13; do
  SSSP_KVAR=$kv timeout 300 python bench.py --config road --steps 16 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | grep -o '"ms_per_step": [0-9.]*' | sed "s/^/kv$kv /"
  done
done
