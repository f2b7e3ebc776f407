#!/bin/bash
# 16-token tiles at mid-size N (fused QKV 6144x2048, Llama v/o 4096x4096, 13B 5120x5120)
cd "$(dirname "$0")/.."
for shape in "6144 2048" "4096 4096" "5120 5120"; do
  for v in "FT2_GEMM_BN=0" "FT2_GEMM_BN=16 FT2_GEMM_SPLITK=2" "FT2_GEMM_BN=16 FT2_GEMM_SPLITK=3" "FT2_GEMM_BN=16 FT2_GEMM_SPLITK=4"; do
    echo "== $shape $v"
    env $v R=24 timeout 120 python tools/insitu_probe.py $shape 2>&1 | grep -E "^\{"
  done
done
