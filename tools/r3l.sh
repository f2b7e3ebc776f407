python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r3l_smoke.txt 2>&1; echo smoke rc $?
FT2_TRACE_CLOCK=1 python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace > /dev/null 2>&1
cp paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace.so paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_trace_clk.so
CLOCK=1 NBLK=24 timeout 120 python tools/b2b_trace.py > gpurun_out/r3l_trace.txt 2>&1; tail -6 gpurun_out/r3l_trace.txt
timeout 1200 python bench.py > gpurun_out/r3l_bench.json 2> gpurun_out/r3l_bench.err; echo bench rc $?
timeout 900 ncu --nvtx --nvtx-include 'ft2_profiled_request/' --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2e_launches.csv python bench.py --profile > gpurun_out/r2e_ncu_list.log 2>&1
python tools/launch_summary.py gpurun_out/r2e_launches.csv > gpurun_out/r2e_launches_summary.txt 2>&1; head -25 gpurun_out/r2e_launches_summary.txt
timeout 900 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include 'ft2_profiled_request/' -k regex:gemm_kernel -s 24 -c 3 -o gpurun_out/r2e_prof_gemm python bench.py --profile > gpurun_out/r2e_ncu_gemm.log 2>&1
python tools/ncu_summary.py gpurun_out/r2e_prof_gemm.ncu-rep > gpurun_out/r2e_ncu_gemm.txt 2>&1; cat gpurun_out/r2e_ncu_gemm.txt | head -40
timeout 600 ncu --set full --clock-control none --import-source on -k regex:'allreduce_protect_kernel|protect_kernel' -c 6 -o gpurun_out/r2e_prof_ar python tools/ar_one.py > gpurun_out/r2e_ncu_ar.log 2>&1
python tools/ncu_summary.py gpurun_out/r2e_prof_ar.ncu-rep > gpurun_out/r2e_ncu_ar.txt 2>&1; head -40 gpurun_out/r2e_ncu_ar.txt
