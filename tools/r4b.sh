# final evidence, end of round 2 (after the out-of-line epilogue helpers and the after-attention L2 prefetch)
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r4b_smoke.txt 2>&1; echo smoke rc $?; tail -2 gpurun_out/r4b_smoke.txt
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r4b_gputests.txt 2>&1; echo tests rc $?; tail -2 gpurun_out/r4b_gputests.txt
timeout 1200 python bench.py > gpurun_out/r4b_bench.json 2> gpurun_out/r4b_bench.err; echo bench rc $?
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r4b_reference.json 2> gpurun_out/r4b_reference.err; echo ref rc $?
timeout 900 ncu --nvtx --nvtx-include 'ft2_profiled_request/' --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2h_launches.csv python bench.py --profile > gpurun_out/r2h_ncu_list.log 2>&1
python tools/launch_summary.py gpurun_out/r2h_launches.csv > gpurun_out/r2h_launches_summary.txt 2>&1; head -12 gpurun_out/r2h_launches_summary.txt
timeout 900 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include 'ft2_profiled_request/' -k regex:gemm_kernel -s 24 -c 3 -o gpurun_out/r2h_prof_gemm python bench.py --profile > gpurun_out/r2h_ncu_gemm.log 2>&1
python tools/ncu_summary.py gpurun_out/r2h_prof_gemm.ncu-rep > gpurun_out/r2h_ncu_gemm.txt 2>&1; grep -E "Kernel Name|time_duration|dram__bytes" gpurun_out/r2h_ncu_gemm.txt
