"""The decode GEMM's opt-in global-memory K split (FT2_GEMM_GSPLIT=1, read
once per process, hence a subprocess): PLAIN within the GEMM tolerance of
the fp64 oracle and the CHECK epilogue bit-exact vs the oracle's R5 on the
kernel's own PLAIN output, as for the default cluster split."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r'''
import sys, numpy as np, torch
sys.path[:0] = [ROOT, ROOT + "/tests"]
import ft2_synth, oracle
import paper_conf_hpdc_sunzmg00y25_b200 as ft2
from gpu_util import dev, host
import ml_dtypes
for (M, N, K) in [(32, 2048, 2048), (17, 1000, 1536), (8, 384, 512)]:
    x = ft2_synth.gen_bf16((M, K), 30, M)
    w = ft2_synth.gen_bf16((N, K), 31, M, scale_log2=ft2_synth.weight_scale_log2(K))
    b = ft2_synth.gen_bf16((N,), 32, M)
    assert ft2.gemm_workspace_bytes(M, N, K) > 0
    y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    ft2.protect_fused_gemm(dev(x), dev(w), y, bias=dev(b), mode=0)
    plain = host(y)
    yr, _ = oracle.linear_f64(x, w, b)
    g = plain.view(ml_dtypes.bfloat16).astype(np.float64)
    rms = np.sqrt(np.mean(yr ** 2, axis=1, keepdims=True))
    assert np.all(np.abs(g - yr) <= 1e-2 * np.maximum(np.abs(yr), 1e-2 * rms)), (M, N, K)
    bnd = np.array([[oracle.f64_to_bf16(-0.2), oracle.f64_to_bf16(0.25)]] * M, np.uint16)
    cnt = torch.zeros(M, dtype=torch.int32, device="cuda")
    y2 = torch.empty_like(y)
    ft2.protect_fused_gemm(dev(x), dev(w), y2, bias=dev(b), mode=1, bounds=dev(bnd), num_seqs=M, corrected_count=cnt)
    ref = plain.copy()
    rc = oracle.protect(ref, bnd, row_to_seq=np.arange(M, dtype=np.int32))
    assert np.array_equal(host(y2), ref) and np.array_equal(cnt.cpu().numpy().astype(np.uint32), rc), (M, N, K)
print("gsplit ok")
'''


def test_gemm_global_split_parity():
    env = dict(os.environ, FT2_GEMM_GSPLIT="1")
    r = subprocess.run([sys.executable, "-c", SCRIPT.replace("ROOT", repr(ROOT))], env=env, capture_output=True,
                       text=True, timeout=600)
    assert r.returncode == 0 and "gsplit ok" in r.stdout, r.stdout[-2000:] + r.stderr[-4000:]
