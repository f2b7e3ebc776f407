python -c "import __graft_entry__ as g; g.build()" > /dev/null
run() { echo "== $1"; for r in 1 2; do env $1 NOTRACE=1 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; done; env $1 NOTRACE=1 SHAPES=2048x2048 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; env $1 NOTRACE=1 SHAPES=4096x4096,4096x4096,11008x4096,4096x11008 NBLK=6 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; }
for t in 3 10 11 12 13 15 16; do run "FT2_GEMM_TRIGGER=$t"; done
run "FT2_GEMM_CTA_CAP=148"
run "FT2_GEMM_W_L2=2"
FT2_TRACE_CLOCK=1 python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace > /dev/null 2>&1
cp paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace.so paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace_clk.so
CLOCK=1 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | tail -5
