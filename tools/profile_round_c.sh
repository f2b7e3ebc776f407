# Round-1 (session c) ncu evidence: launch list of one protected request with
# the SDPA host model, and full captures of the FP32 sweeps and of the fused
# row-parallel all-reduce + check.
set -x
mkdir -p gpurun_out
timeout 900 ncu --nvtx --nvtx-include 'ft2_profiled_request/' --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1c.csv python bench.py --profile > gpurun_out/ncu_list_c.log 2>&1
R=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:'bounds32_kernel|protect32_kernel|allreduce_protect_kernel' -c 4 -o gpurun_out/prof_new_r1c python tools/prot_probe.py > gpurun_out/ncu_new_c.log 2>&1
R=10 timeout 300 python tools/prot_probe.py > gpurun_out/prot_probe_c.txt 2>&1
ls -la gpurun_out
