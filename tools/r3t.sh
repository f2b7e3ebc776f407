python -c "import __graft_entry__ as g; g.build()" > /dev/null
FT2_TRACE_CLOCK=1 python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace > /dev/null 2>&1
cp paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace.so paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace_clk.so
CLOCK=1 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | tail -3
CLOCK=1 SHAPES=2048x2048 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | tail -2
