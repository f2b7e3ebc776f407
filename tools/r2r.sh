python -c "import __graft_entry__ as g; g.build()" > /dev/null
python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace > /dev/null 2>&1
for x in 0 1 0 1; do echo "== XMC=$x"; FT2_GEMM_XMC=$x timeout 120 python tools/b2b_trace.py 2>&1 | head -1; FT2_GEMM_XMC=$x SHAPES=2048x2048 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | head -1; done
for x in 1 0; do FT2_GEMM_XMC=$x FT2_BENCH_SETTLE_MAX_S=30 FT2_BENCH_SKIP=coverage,c2,sweep timeout 900 python bench.py --no-extras --steps 10 > gpurun_out/r2r_x$x.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/r2r_x$x.json').read().strip().splitlines()[-1])
print('xmc $x', round(d['value']), round(d['ms_per_step'],2), {k: round(v) for k,v in d['modes_tokens_per_s'].items() if k!='method'}, round(d['phases']['fused']['decode_ms_per_step'],4), round(d['phases']['off']['decode_ms_per_step'],4))"; done
