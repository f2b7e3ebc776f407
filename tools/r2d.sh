python -c "import __graft_entry__ as g; g.build()" > /dev/null
FT2_TRACE_CLOCK=1 python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace > /dev/null 2>&1
cp paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace.so paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace_clk.so
timeout 900 python -m pytest tests/test_gpu_parity_gemm.py tests/test_gpu_allreduce_protect.py tests/test_gpu_parity_prefill.py -q 2>&1 | tail -3
CLOCK=1 timeout 120 python tools/b2b_trace.py 2>&1 | tail -4
timeout 300 python bench.py --leg c4 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d['value'], d['row_parallel_decode'])"
