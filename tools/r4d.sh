# (no rebuild: libft2.so = BA=64 for N <= 2048 at any K; libft2_base.so = the committed build)
B=$PWD/paper_conf_hpdc_sunzmg00y25_b200/lib/libft2_base.so
run() { echo "== $1"; for r in 1 2; do env $1 NOTRACE=1 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; done; env $1 NOTRACE=1 SHAPES=2048x8192 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; env $1 NOTRACE=1 SHAPES=4096x4096,4096x4096,11008x4096,4096x11008 NBLK=6 timeout 120 python tools/b2b_trace.py 2>&1 | grep graph; }
for k in 1 2; do run "LIBNAME=libft2_base.so"; run "X=1"; done
timeout 1200 python -m pytest tests/test_gpu_parity_gemm.py -q -x 2>&1 | tail -1
for v in "FT2_LIB=$B" "X=1"; do env $v timeout 600 python bench.py --leg models 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$v'[-12:], {k: v['decode_step_us']['fused_check'] for k, v in d.items() if isinstance(v, dict) and 'decode_step_us' in v})"; done
for v in "FT2_LIB=$B" "X=1" "FT2_LIB=$B" "X=1"; do env $v FT2_BENCH_SETTLE_MAX_S=30 FT2_BENCH_SKIP=coverage,c2,sweep timeout 900 python bench.py --no-extras --steps 10 > gpurun_out/r4d_b.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/r4d_b.json').read().strip().splitlines()[-1])
print('$v'[-12:], round(d['value']), round(d['ms_per_step'],2), {k: round(v) for k,v in d['modes_tokens_per_s'].items() if k!='method'}, round(d['phases']['fused']['decode_ms_per_step'],4), round(d['phases']['off']['decode_ms_per_step'],4))"; done
