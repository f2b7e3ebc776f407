python -c "import __graft_entry__ as g; g.build()" > /dev/null
FT2_TRACE_CLOCK=1 python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace > /dev/null 2>&1
cp paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace.so paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace_clk.so
timeout 900 python -m pytest tests/test_gpu_parity_gemm.py tests/test_gpu_c1_pipeline.py tests/test_gpu_parity_fp16.py tests/test_gpu_campaign.py tests/test_gpu_runner_fused_groups.py -q > gpurun_out/r2l_tests.log 2>&1; tail -3 gpurun_out/r2l_tests.log
CLOCK=1 timeout 120 python tools/b2b_trace.py 2>&1 | tail -4
timeout 120 python tools/b2b_trace.py 2>&1 | head -1
for i in 1 2; do FT2_BENCH_SKIP=coverage,c2,sweep timeout 900 python bench.py --no-extras --steps 10 > gpurun_out/r2l_bench$i.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/r2l_bench$i.json').read().strip().splitlines()[-1])
print(round(d['value']), round(d['ms_per_step'],2), {k: round(v) for k,v in d['modes_tokens_per_s'].items() if k!='method'}, round(d['phases']['fused']['decode_ms_per_step'],4), round(d['phases']['fused_plain']['decode_ms_per_step'],4), round(d['phases']['off']['decode_ms_per_step'],4), d['clocks'])"; done
