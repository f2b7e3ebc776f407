python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 1200 python bench.py > gpurun_out/r4g_bench.json 2> gpurun_out/r4g_bench.err; echo bench rc $?
python -c "
import json; d=json.loads(open('gpurun_out/r4g_bench.json').read().strip().splitlines()[-1])
print(round(d['value']), d['roofline']['avg_launch_us'], d['roofline']['frac'], d['roofline']['traffic'], d['roofline']['traffic_note'][:80], d['epilogue_overhead_pct'], d['clocks'])"
