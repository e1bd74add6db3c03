P="import sys,json
for l in sys.stdin:
    d=json.loads(l); print(d['opts'], d['kernel_ms'], d['work_E'])"
for i in 1 2; do
timeout 500 python tools/sweep.py --config road --sources 10 --sets '[{}, {"max_backoff_ns": 256}, {"max_backoff_ns": 128}, {"local_max": 64}, {"active_init": 2}]' 2>&1 | grep kernel_ms | python -c "$P"
done
