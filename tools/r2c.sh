# round-2 session: full GPU tests, host-bound probe, protect ncu capture, default bench
python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/r2c_gpu_tests.log 2>&1; tail -3 gpurun_out/r2c_gpu_tests.log
SECS=20 timeout 200 python tools/host_probe.py > gpurun_out/r2c_host_probe.json 2>&1; tail -c 700 gpurun_out/r2c_host_probe.json; echo
# R=4 timeout 600 ncu --set full --clock-control none -k regex:protect_kernel -s 3 -c 1 -o gpurun_out/r2c_protect python tools/prot_probe.py > gpurun_out/r2c_ncu_protect.log 2>&1
# python tools/ncu_summary.py gpurun_out/r2c_protect.ncu-rep > gpurun_out/r2c_ncu_protect.txt 2>&1; cat gpurun_out/r2c_ncu_protect.txt | head -30
t0=$(date +%s); timeout 1500 python bench.py > gpurun_out/r2c_bench.json 2> gpurun_out/r2c_bench.err; echo "bench wall s: $(( $(date +%s) - t0 ))"; tail -c 300 gpurun_out/r2c_bench.json; tail -3 gpurun_out/r2c_bench.err
