set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
for c in road rmat er; do timeout 600 python bench.py --config $c > gpurun_out/bench_$c.log 2>&1; tail -1 gpurun_out/bench_$c.log; done
timeout 900 bash tools/profile_round.sh r01
ls gpurun_out
