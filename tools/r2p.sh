python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 900 compute-sanitizer --tool racecheck python tools/sanitize_cases.py > gpurun_out/r2p_racecheck.log 2>&1; grep "Race reported" gpurun_out/r2p_racecheck.log | sed 's/(.*//' | sort | uniq -c; tail -2 gpurun_out/r2p_racecheck.log
timeout 600 python -m pytest tests/test_gpu_allreduce_protect.py -q 2>&1 | tail -2
python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace > /dev/null 2>&1
for r in 0 1; do echo "== BA_RULE=$r"; FT2_GEMM_BA_RULE=$r timeout 120 python tools/b2b_trace.py 2>&1 | head -1; FT2_GEMM_BA_RULE=$r timeout 120 python tools/b2b_trace.py 2>&1 | head -1; done
for r in 1 0 1 0; do FT2_GEMM_BA_RULE=$r FT2_BENCH_SKIP=coverage,c2,sweep timeout 900 python bench.py --no-extras --steps 10 > gpurun_out/r2p_b$r.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/r2p_b$r.json').read().strip().splitlines()[-1])
print('rule $r', round(d['value']), round(d['ms_per_step'],2), round(d['phases']['fused']['decode_ms_per_step'],4), round(d['phases']['off']['decode_ms_per_step'],4))"; done
