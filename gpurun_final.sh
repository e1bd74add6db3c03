mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3 > gpurun_out/gpu_tests.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench_road.json 2>gpurun_out/bench_road.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_road.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
for kv in 0 13; do SSSP_KVAR=$kv timeout 300 python bench.py --steps 16 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | grep -o '"ms_per_step": [0-9.]*' | sed "s/^/kv$kv /"; done
cat gpurun_out/gpu_tests.txt gpurun_out/smoke.txt; python -c "import json;d=json.load(open('gpurun_out/bench_road.json'));print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['clocks'],d['e2e']['value'])"
