python -c "import __graft_entry__ as g; g.build()" > /dev/null
FT2_TRACE_CLOCK=1 python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace > /dev/null 2>&1
cp paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace.so paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace_clk.so
timeout 900 python -m pytest tests/test_gpu_parity_gemm.py -q > gpurun_out/r2m_tests.log 2>&1; tail -2 gpurun_out/r2m_tests.log
CLOCK=1 timeout 120 python tools/b2b_trace.py 2>&1 | tail -3; timeout 120 python tools/b2b_trace.py 2>&1 | head -1; SAMEW=1 SHAPES=2048x2048 NBLK=24 CLOCK=1 timeout 120 python tools/b2b_trace.py 2>&1 | tail -1
SHAPES=4096x4096,11008x4096,4096x11008 NBLK=6 timeout 120 python tools/b2b_trace.py 2>&1 | head -1
