timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -1
for i in 1 2; do timeout 300 python bench.py --steps 8 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import sys,json;d=json.loads(sys.stdin.read());print(d['ms_per_step'],d['value'],d['e2e']['value'])"; done
