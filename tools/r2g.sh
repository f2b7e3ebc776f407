python -c "import __graft_entry__ as g; g.build()" > /dev/null
for ba in 64 128 64 128; do
  FT2_GEMM_BA=$ba FT2_BENCH_SKIP=coverage,c2,sweep timeout 900 python bench.py --no-extras --steps 10 > gpurun_out/r2g_bench_ba$ba.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/r2g_bench_ba$ba.json').read().strip().splitlines()[-1])
print('BA=$ba', round(d['value']), round(d['ms_per_step'],2), {k: round(v) for k,v in d['modes_tokens_per_s'].items() if k!='method'}, round(d['phases']['fused']['decode_ms_per_step'],4), round(d['phases']['fused_plain']['decode_ms_per_step'],4), round(d['phases']['off']['decode_ms_per_step'],4))"
done
for ba in 64 128; do FT2_GEMM_BA=$ba timeout 600 python bench.py --leg c3 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('c3 BA=$ba', {k: (v['us'], round(v['roofline']['frac'],3)) for k,v in d['shapes'].items()})"; done
