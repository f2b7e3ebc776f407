#!/bin/bash
# In-situ decode GEMM (layer_norm -> linear pairs in a CUDA graph) at the OPT-1.3B
# v/out_proj shape for several split-K factors (0 = planner): does keeping every
# cluster resident in one wave (max_clusters >= tiles) beat the deeper split?
cd "$(dirname "$0")/.."
for sk in 0 4 5 6 8; do
  echo "== FT2_GEMM_SPLITK=$sk"
  FT2_GEMM_SPLITK=$sk R=48 timeout 120 python tools/insitu_probe.py 2048 2048 2>&1 | grep -E "^\{"
done
