python -c "import __graft_entry__ as g; g.build()" > /dev/null
run() { echo "== $1"; for r in 1 2; do env $1 NOTRACE=1 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; done; env $1 NOTRACE=1 SHAPES=2048x2048 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; env $1 NOTRACE=1 SHAPES=4096x4096,4096x4096,11008x4096,4096x11008 NBLK=6 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; }
run "FT2_GEMM_TRIGGER=1"; run "FT2_GEMM_TRIGGER=2"; run "FT2_GEMM_TRIGGER=3"
for v in 1 2 3 1 2 3; do FT2_GEMM_TRIGGER=$v FT2_BENCH_SETTLE_MAX_S=30 FT2_BENCH_SKIP=coverage,c2,sweep timeout 900 python bench.py --no-extras --steps 10 > gpurun_out/r3n_b.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/r3n_b.json').read().strip().splitlines()[-1])
print('TRIGGER $v', round(d['value']), round(d['ms_per_step'],2), {k: round(v) for k,v in d['modes_tokens_per_s'].items() if k!='method'}, round(d['phases']['fused']['decode_ms_per_step'],4), round(d['phases']['off']['decode_ms_per_step'],4))"; done
for v in 1 2; do FT2_GEMM_TRIGGER=$v timeout 600 python bench.py --leg c3 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('c3 TRIGGER $v', {k: v['us'] for k, v in d.get('shapes', {}).items()})"; done
