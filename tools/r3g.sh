python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 600 python -m pytest tests/test_gpu_allreduce_protect.py -q 2>&1 | tail -2
timeout 600 python bench.py --leg c4 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d.get('row_parallel_decode'); r.pop('variants',None); print(json.dumps(r))"
run() { echo "== $1"; for r in 1 2; do env $1 NOTRACE=1 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; done; env $1 NOTRACE=1 SHAPES=2048x2048 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; env $1 NOTRACE=1 SHAPES=4096x4096,4096x4096,11008x4096,4096x11008 NBLK=6 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; }
run "FT2_GEMM_MMA2=0"
run "FT2_GEMM_MMA2=1"
run "FT2_GEMM_MMA2=0"
run "FT2_GEMM_MMA2=1"
FT2_GEMM_MMA2=1 timeout 900 python -m pytest tests/test_gpu_parity_gemm.py -q -x > gpurun_out/r3g_mma2_tests.log 2>&1; tail -2 gpurun_out/r3g_mma2_tests.log
for w in 0 1; do FT2_GEMM_MMA2=$w FT2_BENCH_SETTLE_MAX_S=30 FT2_BENCH_SKIP=coverage,c2,sweep timeout 900 python bench.py --no-extras --steps 10 > gpurun_out/r3g_b$w.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/r3g_b$w.json').read().strip().splitlines()[-1])
print('MMA2 $w', round(d['value']), round(d['ms_per_step'],2), {k: round(v) for k,v in d['modes_tokens_per_s'].items() if k!='method'}, round(d['phases']['fused']['decode_ms_per_step'],4), round(d['phases']['off']['decode_ms_per_step'],4))"; done
