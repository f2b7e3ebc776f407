#!/bin/bash
cd "$(dirname "$0")/.."
for shape in "6144 2048" "5120 5120" "5120 13824" "4608 2048"; do
  for sk in 0 5 6 7; do
    echo "== $shape FT2_GEMM_SPLITK=$sk"
    FT2_GEMM_SPLITK=$sk R=24 timeout 120 python tools/insitu_probe.py $shape 2>&1 | grep -E "^\{"
  done
done
