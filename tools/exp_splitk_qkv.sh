#!/bin/bash
# In-situ decode GEMM at the fused-QKV shape of OPT-1.3B (N = 6144, K = 2048)
# for split-K 1..6 (0 = planner): cluster residency vs split depth.
cd "$(dirname "$0")/.."
for sk in 0 2 3 4 6; do
  echo "== FT2_GEMM_SPLITK=$sk"
  FT2_GEMM_SPLITK=$sk R=48 timeout 120 python tools/insitu_probe.py 6144 2048 2>&1 | grep -E "^\{"
done
FT2_GEMM_DEBUG=1 R=2 timeout 60 python tools/insitu_probe.py 6144 2048 2>&1 | grep "ft2 gemm" | head -1
