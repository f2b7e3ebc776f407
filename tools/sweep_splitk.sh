for sh in "32 11008 4096" "32 4096 4096" "32 2048 2048" "32 4096 11008" "32 2048 8192" "1 2048 2048" "32 8192 2048"; do
  FT2_GEMM_DEBUG=1 R=20 timeout 60 python tools/gemm_probe.py $sh 2>&1 | grep -E "ft2 gemm|cublas" | head -2
  for sk in 1 2 3 4 6 8 12 16; do echo -n "sk=$sk "; FT2_GEMM_SPLITK=$sk R=20 timeout 60 python tools/gemm_probe.py $sh 2>&1 | grep cublas; done
done
