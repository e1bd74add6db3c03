mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "perturbation or star or scaled or golden or full_size" > gpurun_out/pytest4.log 2>&1; echo pytest=$? >> gpurun_out/pytest4.log
for c in road rmat er; do timeout 600 python tools/sweep.py --config $c --sources 6 --profile --sets '[{}, {"split_degree": 4294967295}]' > gpurun_out/sw4_$c.log 2>&1; done
timeout 600 python tools/sweep.py --config rmat --sources 6 --profile --sets '[{"split_degree": 2048}, {"split_degree": 8192}, {"split_degree": 16384}]' --deltas 3 >> gpurun_out/sw4_rmat.log 2>&1
timeout 300 python tools/trace.py --config road --rows 40 > gpurun_out/trace4_road.log 2>&1
