mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3 > gpurun_out/gpu_tests.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench_road.json 2>gpurun_out/bench_road.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_road.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
P="import sys,json
for l in sys.stdin:
    d=json.loads(l); print(d['opts'], d['kernel_ms'], d['work_E'], d['final_k'][:4])"
for i in 1 2; do timeout 500 python tools/sweep.py --config road --sources 10 --sets '[{}, {"active_init": 1}, {"active_init": 3}]' 2>&1 | grep kernel_ms | python -c "$P" >> gpurun_out/sweep31.txt; done
cat gpurun_out/gpu_tests.txt gpurun_out/smoke.txt gpurun_out/sweep31.txt; python -c "import json;d=json.load(open('gpurun_out/bench_road.json'));print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['clocks'],d['e2e']['value'],d['work_efficiency'])"
