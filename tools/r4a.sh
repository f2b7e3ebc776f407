python -c "import __graft_entry__ as g; g.build()" > /dev/null
for v in 0 2 0 2 1; do FT2_L2_PREFETCH=$v FT2_BENCH_SETTLE_MAX_S=30 FT2_BENCH_SKIP=coverage,c2,sweep timeout 900 python bench.py --no-extras --steps 10 > gpurun_out/r4a_b.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/r4a_b.json').read().strip().splitlines()[-1])
print('PF $v', round(d['value']), round(d['ms_per_step'],2), {k: round(v) for k,v in d['modes_tokens_per_s'].items() if k!='method'}, round(d['phases']['fused']['decode_ms_per_step'],4), round(d['phases']['off']['decode_ms_per_step'],4))"; done
FT2_L2_PREFETCH=2 timeout 900 python -m pytest tests/test_gpu_runner_fused_groups.py tests/test_gpu_c1_pipeline.py -q -x 2>&1 | tail -1
