python -c "import __graft_entry__ as g; g.build()" > /dev/null
./tools/mma_probe 2>&1 | head -8 > gpurun_out/r3e_mma_mw.txt; cat gpurun_out/r3e_mma_mw.txt
run() { echo "== $1"; for r in 1 2; do env $1 NOTRACE=1 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; done; env $1 NOTRACE=1 SHAPES=4096x4096,4096x4096,11008x4096,4096x11008 NBLK=6 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; }
run "FT2_GEMM_W_L2=0"
run "FT2_GEMM_W_L2=1"
run "FT2_GEMM_W_L2=2"
run "FT2_GEMM_W_L2=2 FT2_GEMM_BA=128 FT2_GEMM_BN=32"
run "FT2_GEMM_W_L2=0"
for w in 0 2; do FT2_GEMM_W_L2=$w FT2_BENCH_SETTLE_MAX_S=30 FT2_BENCH_SKIP=coverage,c2,sweep timeout 900 python bench.py --no-extras --steps 10 > gpurun_out/r3e_b$w.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/r3e_b$w.json').read().strip().splitlines()[-1])
print('W_L2 $w', round(d['value']), round(d['ms_per_step'],2), {k: round(v) for k,v in d['modes_tokens_per_s'].items() if k!='method'}, round(d['phases']['fused']['decode_ms_per_step'],4), round(d['phases']['off']['decode_ms_per_step'],4))"; done
timeout 600 python -m pytest tests/test_gpu_allreduce_protect.py -q 2>&1 | tail -1
timeout 600 python bench.py --leg c4 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps(d.get('row_parallel_decode')))"
