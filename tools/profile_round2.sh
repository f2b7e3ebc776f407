# Round-2 ncu evidence: launch list of one protected request (OPT-1.3B, B=32,
# fused), full captures of the decode GEMM (v/out at BA=64, fc2 at BA=128) in
# that request, of the bounds sweep in its prefill, and of one 2048x2048 GEMM
# launch alone.
python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 900 ncu --nvtx --nvtx-include 'ft2_profiled_request/' --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2_launches.csv python bench.py --profile > gpurun_out/r2_ncu_list.log 2>&1
python tools/launch_summary.py gpurun_out/r2_launches.csv > gpurun_out/r2_launches_summary.txt 2>&1; head -25 gpurun_out/r2_launches_summary.txt
timeout 900 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include 'ft2_profiled_request/' -k regex:gemm_kernel -s 24 -c 3 -o gpurun_out/r2_prof_gemm python bench.py --profile > gpurun_out/r2_ncu_gemm.log 2>&1
python tools/ncu_summary.py gpurun_out/r2_prof_gemm.ncu-rep > gpurun_out/r2_ncu_gemm.txt 2>&1; cat gpurun_out/r2_ncu_gemm.txt
timeout 600 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include 'ft2_profiled_request/' -k regex:bounds_kernel -c 2 -o gpurun_out/r2_prof_bounds python bench.py --profile > gpurun_out/r2_ncu_bounds.log 2>&1
python tools/ncu_summary.py gpurun_out/r2_prof_bounds.ncu-rep > gpurun_out/r2_ncu_bounds.txt 2>&1; cat gpurun_out/r2_ncu_bounds.txt | head -25
