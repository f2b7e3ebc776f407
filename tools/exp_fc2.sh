#!/bin/bash
# OPT-1.3B fc2 decode shape (2048 x 8192, M = 32): split-K / token-tile sweep
cd "$(dirname "$0")/.."
FT2_GEMM_DEBUG=1 R=2 timeout 60 python tools/insitu_probe.py 2048 8192 2>&1 | grep "ft2 gemm" | head -1
for v in "FT2_GEMM_SPLITK=0" "FT2_GEMM_SPLITK=10" "FT2_GEMM_SPLITK=14" "FT2_GEMM_SPLITK=16" "FT2_GEMM_BN=16 FT2_GEMM_SPLITK=8" "FT2_GEMM_BN=16 FT2_GEMM_SPLITK=12"; do
  echo "== $v"
  env $v R=48 timeout 120 python tools/insitu_probe.py 2048 8192 2>&1 | grep -E "^\{"
done
