python -c "import __graft_entry__ as g; g.build()" > /dev/null
FT2_TRACE_CLOCK=1 python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace > /dev/null 2>&1
cp paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace.so paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace_clk.so
python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace > /dev/null 2>&1
for sp in 0 1; do echo "== SPREAD=$sp"; FT2_GEMM_SPREAD=$sp timeout 120 python tools/b2b_trace.py 2>&1 | grep -E "graph|SM sharing|Error"; FT2_GEMM_SPREAD=$sp SHAPES=2048x2048 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep -E "graph|SM sharing"; done
echo "== SPREAD=0 CLOCK"; CLOCK=1 timeout 120 python tools/b2b_trace.py 2>&1 | tail -4
echo "== SPREAD=1 CLOCK"; FT2_GEMM_SPREAD=1 CLOCK=1 timeout 120 python tools/b2b_trace.py 2>&1 | tail -4
echo "== NACC=4"; FT2_GEMM_NACC=4 timeout 120 python tools/b2b_trace.py 2>&1 | grep -E "graph"
echo "== SMEM_PAD=20000 (one CTA per SM)"; FT2_GEMM_SMEM_PAD=20000 timeout 120 python tools/b2b_trace.py 2>&1 | grep -E "graph|SM sharing"
