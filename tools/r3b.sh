python -c "import __graft_entry__ as g; g.build()" > /dev/null
./tools/mma_probe > gpurun_out/r3b_mma_probe.txt 2>&1; cat gpurun_out/r3b_mma_probe.txt
for n in 1 4 2 1 4; do echo "== NACC=$n"; FT2_GEMM_NACC=$n timeout 120 python tools/b2b_trace.py 2>&1 | head -1; FT2_GEMM_NACC=$n SHAPES=2048x2048 NBLK=24 timeout 120 python tools/b2b_trace.py 2>&1 | head -1; FT2_GEMM_NACC=$n SHAPES=4096x4096,11008x4096,4096x11008 NBLK=6 timeout 120 python tools/b2b_trace.py 2>&1 | head -1; done
FT2_GEMM_NACC=4 timeout 900 python -m pytest tests/test_gpu_parity_gemm.py -q -x > gpurun_out/r3b_nacc4_tests.log 2>&1; tail -2 gpurun_out/r3b_nacc4_tests.log
timeout 600 python -m pytest tests/test_gpu_allreduce_protect.py -q 2>&1 | tail -2
for p in 1 0 1; do FT2_AR_PDL=$p timeout 600 python bench.py --leg c4 > gpurun_out/r3b_c4_pdl$p.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/r3b_c4_pdl$p.json').read().strip().splitlines()[-1]); print('AR_PDL=$p', json.dumps(d.get('row_parallel_decode', d))[:400])"; done
