#!/bin/bash
# In-situ decode GEMM (layer_norm -> linear pairs in a CUDA graph) at the OPT-1.3B
# v/out_proj shape for several split-K factors (0 = planner).
cd "$(dirname "$0")/.."
FT2_GEMM_DEBUG=1 R=2 timeout 60 python tools/insitu_probe.py 2048 2048 2>&1 | grep "ft2 gemm" | head -1
for sk in 0 8 9 10 11 12; do
  echo "== FT2_GEMM_SPLITK=$sk"
  FT2_GEMM_SPLITK=$sk R=48 timeout 120 python tools/insitu_probe.py 2048 2048 2>&1 | grep -E "^\{"
done
