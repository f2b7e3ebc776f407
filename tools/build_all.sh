#!/bin/bash
# Build libft2.so and the trace variant; exit non-zero on any compiler error.
set -e
cd "$(dirname "$0")/.."
out=$(python -m paper_conf_hpdc_sunzmg00y25_b200.build 2>&1) || { echo "$out"; exit 1; }
echo "$out" | grep -E "error|warning" && exit 1
out=$(FT2_TRACE_CLOCK=1 python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace 2>&1) || { echo "$out"; exit 1; }
echo "build ok"
