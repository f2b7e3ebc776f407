#!/bin/bash
# In-situ and back-to-back decode GEMM at mid-size N (Llama v/o 4096x4096, fused
# OPT QKV 6144x2048, Llama down 4096x11008) for several split-K factors.
cd "$(dirname "$0")/.."
for shape in "4096 4096" "6144 2048" "4096 11008"; do
  for sk in 0 4 5 6 8; do
    echo "== $shape FT2_GEMM_SPLITK=$sk"
    FT2_GEMM_SPLITK=$sk R=24 timeout 120 python tools/insitu_probe.py $shape 2>&1 | grep -E "^\{"
  done
done
