# in-situ GEMM experiments (env knobs of gemm_sm100.cu); usage: bash tools/exp_insitu.sh
CLOCK=1 timeout 120 python tools/gap_probe.py 2048 2048 2>&1 | grep -E "cycles"; timeout 120 python tools/gap_probe.py 2048 2048 2>&1 | grep -E "ft2|cublas"
timeout 120 python tools/insitu_probe.py 2048 2048 | tail -1
timeout 120 python tools/insitu_probe.py | tail -1
