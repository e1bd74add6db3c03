P="import sys,json
for l in sys.stdin:
    d=json.loads(l); print(d['config'], d['opts'], d['kernel_ms'], d['work_E'], d['final_k'][:4])"
for i in 1 2; do
for e in 0 0x20000; do
for c in road rmat er; do
echo "EXP=$e"; SSSP_EXP=$e timeout 300 python tools/sweep.py --config $c --sources 12 --sets '[{}]' 2>&1 | grep kernel_ms | python -c "$P"
done; done; done
timeout 600 python -m pytest tests -m gpu -x -q -k "road or grid or rmat or er" 2>&1 | tail -2
