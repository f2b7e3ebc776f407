#!/bin/bash
# Decode GEMM at M = 32 with 16-token tiles (two token tiles per feature tile):
# more, smaller clusters that all fit in one wave, vs the default 32-token tile.
cd "$(dirname "$0")/.."
for shape in "2048 2048" "2048 8192"; do
  for v in "FT2_GEMM_BN=0" "FT2_GEMM_BN=16" "FT2_GEMM_BN=16 FT2_GEMM_SPLITK=4" "FT2_GEMM_BN=16 FT2_GEMM_SPLITK=6"; do
    echo "== $shape $v"
    env $v R=48 timeout 120 python tools/insitu_probe.py $shape 2>&1 | grep -E "^\{"
  done
done
