python -c "import __graft_entry__ as g; g.build()" > /dev/null
run() { echo "== $1"; for r in 1 2; do env $1 NOTRACE=1 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; done; env $1 NOTRACE=1 SHAPES=2048x8192 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; }
for k in 1 2; do run "X=1"; run "FT2_GEMM_CTA_CAP=148"; run "FT2_GEMM_CTA_CAP=192"; done
for v in "X=1" "FT2_GEMM_CTA_CAP=148" "X=1" "FT2_GEMM_CTA_CAP=148"; do env $v FT2_BENCH_SETTLE_MAX_S=30 FT2_BENCH_SKIP=coverage,c2,sweep timeout 900 python bench.py --no-extras --steps 10 > gpurun_out/r4h_b.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/r4h_b.json').read().strip().splitlines()[-1])
print('$v'[-20:], round(d['value']), round(d['ms_per_step'],2), {k: round(v) for k,v in d['modes_tokens_per_s'].items() if k!='method'}, round(d['phases']['fused']['decode_ms_per_step'],4), round(d['phases']['off']['decode_ms_per_step'],4))"; done
