set -x
timeout 300 python tools/prefill_gemm_probe.py > gpurun_out/prefill_gemm.txt 2>&1
timeout 900 ncu --nvtx --nvtx-include 'ft2_profiled_request/' --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1b.csv python bench.py --profile > gpurun_out/ncu_list.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include 'ft2_profiled_request/' -k regex:gemm_kernel -s 24 -c 3 -o gpurun_out/prof_gemm_r1b python bench.py --profile > gpurun_out/ncu_gemm.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include 'ft2_profiled_request/' -k regex:bounds_kernel -c 2 -o gpurun_out/prof_bounds_r1b python bench.py --profile > gpurun_out/ncu_bounds.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:'bounds_kernel|protect_kernel' -c 2 -o gpurun_out/prof_prot_r1b python tools/prot_probe.py > gpurun_out/ncu_prot.log 2>&1
ls -la gpurun_out
