python -c "import __graft_entry__ as g; g.build()" > /dev/null
for v in 1 3 1 3; do FT2_GEMM_TRIGGER=$v timeout 600 python bench.py --leg c3 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('c3 TRIGGER $v', {k: (v['us']['plain'], v['us']['check']) for k, v in d.get('shapes', {}).items()})"; done
for v in 1 3; do FT2_GEMM_TRIGGER=$v timeout 600 python bench.py --leg models 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); m=d.get('models', d); print('models TRIGGER $v', json.dumps(m)[:1500])"; done
FT2_GEMM_TRIGGER=3 timeout 1200 python -m pytest tests/test_gpu_parity_gemm.py tests/test_gpu_runner_fused_groups.py -q -x 2>&1 | tail -1
