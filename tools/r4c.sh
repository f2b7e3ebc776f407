python -c "import __graft_entry__ as g; g.build()" > /dev/null
for v in 0 2; do FT2_L2_PREFETCH=$v FT2_BENCH_SKIP=coverage,c2,sweep,partitioned timeout 900 python bench.py --steps 3 > gpurun_out/r4c_pf$v.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/r4c_pf$v.json').read().strip().splitlines()[-1])
print('PF $v', round(d['value']), d['roofline']['avg_launch_us'], d['roofline']['frac'], d['roofline']['l2_prefetch_hint'])"; done
timeout 1200 python bench.py > gpurun_out/r4c_bench.json 2> gpurun_out/r4c_bench.err; echo bench rc $?
python -c "
import json; d=json.loads(open('gpurun_out/r4c_bench.json').read().strip().splitlines()[-1])
print(round(d['value']), d['roofline']['avg_launch_us'], d['roofline']['frac'], d['epilogue_overhead_pct'], d['clocks'])"
