python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 600 python -m pytest tests/test_gpu_allreduce_protect.py -q 2>&1 | tail -2
for p in 1 0; do FT2_AR_PDL=$p timeout 600 python bench.py --leg c4 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d.get('row_parallel_decode'); r.pop('variants',None); print('PDL $p', json.dumps(r))"; done
