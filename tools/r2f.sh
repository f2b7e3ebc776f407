python -c "import __graft_entry__ as g; g.build()" > /dev/null
FT2_TRACE_CLOCK=1 python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace > /dev/null 2>&1
cp paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace.so paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace_clk.so
FT2_GEMM_BA=64 timeout 600 python -m pytest tests/test_gpu_parity_gemm.py -q -x -k "plain_within or epilogue_bit_exact or masks or overflow" 2>&1 | tail -4
for ba in 128 64; do echo "== BA=$ba"; FT2_GEMM_BA=$ba FT2_GEMM_DEBUG=1 CLOCK=1 timeout 120 python tools/b2b_trace.py 2>&1 | grep -v "^\[ft2" | tail -4; FT2_GEMM_BA=$ba FT2_GEMM_DEBUG=1 CLOCK=1 timeout 120 python tools/b2b_trace.py 2>&1 | grep "^\[ft2" | sort -u; done
