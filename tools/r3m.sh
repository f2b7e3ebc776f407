python -c "import __graft_entry__ as g; g.build()" > /dev/null
run() { echo "== $1"; for r in 1 2; do env $1 NOTRACE=1 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; done; env $1 NOTRACE=1 SHAPES=2048x2048 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; env $1 NOTRACE=1 SHAPES=4096x4096,4096x4096,11008x4096,4096x11008 NBLK=6 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; }
for k in 1 2; do
run "X=1"
run "FT2_GEMM_TRIGGER=2"
run "FT2_GEMM_BA=128 FT2_GEMM_BN=32"
run "FT2_GEMM_BA=128 FT2_GEMM_BN=32 FT2_GEMM_MMA2=2"
run "FT2_GEMM_MMA2=2"
done
FT2_GEMM_BA=128 FT2_GEMM_BN=32 FT2_GEMM_MMA2=2 timeout 1200 python -m pytest tests/test_gpu_parity_gemm.py -q -x 2>&1 | tail -1
FT2_GEMM_MMA2=2 timeout 1200 python -m pytest tests/test_gpu_parity_gemm.py -q -x 2>&1 | tail -1
