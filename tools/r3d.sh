python -c "import __graft_entry__ as g; g.build()" > /dev/null
python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace > /dev/null 2>&1
run() { echo "== $1"; for r in 1 2; do env $1 NOTRACE=1 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; done; env $1 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep "SM sharing"; env $1 NOTRACE=1 SHAPES=4096x4096,4096x4096,11008x4096,4096x11008 NBLK=6 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; }
run "X=0"
run "FT2_GEMM_CTA_CAP=148"
run "FT2_GEMM_CTA_CAP=128"
run "FT2_GEMM_BA=128 FT2_GEMM_BN=32"
run "FT2_GEMM_BA=128 FT2_GEMM_BN=32 FT2_GEMM_CTA_CAP=148"
run "FT2_GEMM_BA=128 FT2_GEMM_BN=32 FT2_GEMM_CTA_CAP=128"
run "FT2_GEMM_CTA_CAP=160"
run "X=0"
