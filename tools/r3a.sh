python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r3a_smoke.txt 2>&1; echo smoke rc $?
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r3a_gputests.txt 2>&1; echo tests rc $?; tail -3 gpurun_out/r3a_gputests.txt
timeout 900 python bench.py > gpurun_out/r3a_bench.json 2> gpurun_out/r3a_bench.err; echo bench rc $?
tail -c 600 gpurun_out/r3a_bench.json
