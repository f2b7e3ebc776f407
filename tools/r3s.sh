python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 1500 python -m pytest tests/test_gpu_parity_prefill.py -q -x > gpurun_out/r3s_prefill_tests.log 2>&1; echo tests rc $?; tail -3 gpurun_out/r3s_prefill_tests.log
for s in 0 -1; do echo "== FT2_PREFILL_SPLITS=$s"; FT2_PREFILL_SPLITS=$s timeout 300 python tools/prefill_gemm_probe.py 2>&1 | tail -8; done
for s in 0 -1; do FT2_PREFILL_SPLITS=$s FT2_GEMM_SWAP_MAX=128 timeout 300 python tools/m256_probe.py 2>&1 | tail -1; done
