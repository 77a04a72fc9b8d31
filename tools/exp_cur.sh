timeout 900 python -m pytest tests -m gpu -q --timeout 300 2>&1 | tail -1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 300 python bench.py 2>/dev/null | cut -c1-200
timeout 300 python bench.py --N 32 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print('N32', d['us_per_spmm'], d['roofline']['frac'])"
