python -c "import __graft_entry__ as g; g.build()" > /dev/null
FT2_TRACE_CLOCK=1 python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace > /dev/null 2>&1
cp paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace.so paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace_clk.so
timeout 900 python -m pytest tests/test_gpu_parity_gemm.py tests/test_gpu_c1_pipeline.py tests/test_gpu_runner_fused_groups.py tests/test_gpu_parity_fp16.py -q -x 2>&1 | tail -3
for x in 0 1; do echo "== XMC=$x"; FT2_GEMM_XMC=$x FT2_GEMM_DEBUG=1 CLOCK=1 timeout 120 python tools/b2b_trace.py 2>&1 | grep -v "^\[ft2" | tail -3; FT2_GEMM_XMC=$x FT2_GEMM_DEBUG=1 CLOCK=1 timeout 120 python tools/b2b_trace.py 2>&1 | grep "^\[ft2" | sort -u; done
for x in 1 0; do FT2_GEMM_XMC=$x timeout 600 python bench.py --leg c3 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('c3 XMC=$x', {k: (v['us']['check'], round(v['roofline']['frac'],3)) for k,v in d['shapes'].items()})"; done
