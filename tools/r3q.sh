python -c "import __graft_entry__ as g; g.build()" > /dev/null
for s in 0 -1 2 3 4; do echo "== FT2_PREFILL_SPLITS=$s"; FT2_PREFILL_SPLITS=$s SMALL=1 timeout 300 python tools/prefill_gemm_probe.py 2>&1 | tail -3; done
