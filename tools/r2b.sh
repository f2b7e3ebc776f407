python -c "import __graft_entry__ as g; g.build()" > /dev/null
python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace > /dev/null 2>&1
run() { echo "== $*"; env "$@" timeout 120 python tools/b2b_trace.py 2>&1 | grep "graph of"; }
run PF=0
run PF=1
run PF=1 FT2_GEMM_PF_AT=0
run PF=0 SHAPES=4096x4096,11008x4096,4096x11008 NBLK=6
run PF=1 SHAPES=4096x4096,11008x4096,4096x11008 NBLK=6
run PF=0 SHAPES=6144x2048,2048x2048,2048x8192
run PF=1 SHAPES=6144x2048,2048x2048,2048x8192
for pf in 0 1; do echo "== bench FT2_L2_PREFETCH=$pf"; FT2_L2_PREFETCH=$pf timeout 600 python bench.py --no-extras --steps 10 > gpurun_out/r2_bench_pf$pf.json 2>gpurun_out/r2_bench_pf$pf.err; python -c "
import json; d=json.loads(open('gpurun_out/r2_bench_pf$pf.json').read().strip().splitlines()[-1]); print(round(d['value']), round(d['ms_per_step'],2), {k: round(v) for k,v in d['modes_tokens_per_s'].items() if k!='method'}, d['phases']['fused'], d['phases']['fused_plain'], d['phases']['off'])"; done
