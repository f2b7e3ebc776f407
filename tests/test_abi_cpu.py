"""The C-ABI library loads and exports every symbol include/ft2.h declares;
argument validation behaves as documented (no GPU needed: every case here
returns before any CUDA call)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    from paper_conf_hpdc_sunzmg00y25_b200 import build as b
    b.build()
    from paper_conf_hpdc_sunzmg00y25_b200 import _lib
    return _lib.load()


def _declared():
    src = open(os.path.join(ROOT, "include", "ft2.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(ft2_[a-z0-9_]+)\s*\(", src)))


def test_every_declared_symbol_is_exported(L):
    decl = _declared()
    assert len(decl) >= 10
    for name in decl:
        assert hasattr(L, name), name
    from paper_conf_hpdc_sunzmg00y25_b200 import _lib
    assert sorted(_lib.EXPORTS) == decl


def test_status_strings_and_version(L):
    assert L.ft2_status_string(0) == b"FT2_OK"
    assert L.ft2_status_string(4) == b"FT2_ERR_CUDA"
    assert L.ft2_version().startswith(b"ft2-b200")


def test_workspace_bytes(L):
    assert L.ft2_workspace_bytes(1) >= 4 * 7
    assert L.ft2_workspace_bytes(1000) > L.ft2_workspace_bytes(1)


def test_validation_without_gpu(L):
    from paper_conf_hpdc_sunzmg00y25_b200._lib import (FT2_ERR_INVALID_ARG, FT2_ERR_MISALIGNED,
                                                        FT2_ERR_UNSUPPORTED, FT2_OK, Tensor)
    P = ctypes.c_void_p
    good = Tensor(0x1000, 4, 16, 16, 0)
    # NULL bounds / num_seqs < 1
    assert L.ft2_protect(good, None, None, 1, None, None) == FT2_ERR_INVALID_ARG
    assert L.ft2_protect(good, None, P(0x2000), 0, None, None) == FT2_ERR_INVALID_ARG
    # ld < n, negative rows
    assert L.ft2_protect(Tensor(0x1000, 4, 16, 8, 0), None, P(0x2000), 1, None, None) == FT2_ERR_INVALID_ARG
    assert L.ft2_protect(Tensor(0x1000, -1, 16, 16, 0), None, P(0x2000), 1, None, None) == FT2_ERR_INVALID_ARG
    # misaligned base, n % 8
    assert L.ft2_protect(Tensor(0x1002, 4, 16, 16, 0), None, P(0x2000), 1, None, None) == FT2_ERR_MISALIGNED
    assert L.ft2_protect(Tensor(0x1000, 4, 12, 16, 0), None, P(0x2000), 1, None, None) == FT2_ERR_MISALIGNED
    # unknown dtype; FP32 (16-byte vectors of 4): n % 4, fp32 bounds 8-byte aligned
    assert L.ft2_protect(Tensor(0x1000, 4, 16, 16, 3), None, P(0x2000), 1, None, None) == FT2_ERR_UNSUPPORTED
    assert L.ft2_protect(Tensor(0x1000, 4, 6, 8, 2), None, P(0x2000), 1, None, None) == FT2_ERR_MISALIGNED
    assert L.ft2_protect(Tensor(0x1000, 4, 8, 10, 2), None, P(0x2000), 1, None, None) == FT2_ERR_MISALIGNED
    assert L.ft2_protect(Tensor(0x1000, 4, 8, 8, 2), None, P(0x2004), 1, None, None) == FT2_ERR_MISALIGNED
    assert L.ft2_bounds_finalize(P(0x1000), 1, 2.0, 3, P(0x2000), None) == FT2_ERR_UNSUPPORTED
    # the fused GEMMs are bf16/fp16 tensor-core contractions: FP32 is unsupported
    assert L.ft2_protect_fused_gemm(P(0x1000), 16, P(0x2000), 16, None, P(0x3000), 16, 4, 16, 16, 0, 2, 0, 16,
                                    None, None, 0, None, None, 0, 0, 0, None, None, 0, None) == FT2_ERR_UNSUPPORTED
    # zero-size -> OK with no launch
    n0 = L.ft2_launch_count()
    assert L.ft2_protect(Tensor(0x1000, 0, 16, 16, 0), None, P(0x2000), 1, None, None) == FT2_OK
    assert L.ft2_launch_count() == n0
    # row_to_seq NULL needs num_seqs in {1, rows}
    assert L.ft2_protect(good, None, P(0x2000), 3, None, None) == FT2_ERR_INVALID_ARG
    # bounds: scale < 1, non-finite, missing workspace, correct without finalize
    args = dict(so=None, S=1, fin=1, cor=0, b=P(0x3000), k=None, nf=None, ws=P(0x4000))
    def bfp(scale, **kw):
        a = dict(args, **kw)
        return L.ft2_bounds_from_prefill(good, a["so"], a["S"], scale, a["fin"], a["cor"], a["b"], a["k"], a["nf"],
                                         None, a["ws"], None)
    assert bfp(0.5) == FT2_ERR_INVALID_ARG
    assert bfp(float("nan")) == FT2_ERR_INVALID_ARG
    assert bfp(2.0, ws=None) == FT2_ERR_INVALID_ARG
    assert bfp(2.0, fin=0, cor=1, k=P(0x5000)) == FT2_ERR_INVALID_ARG
    assert bfp(2.0, S=2) == FT2_ERR_INVALID_ARG       # several sequences need seq_offsets
    # fused gemm: misaligned K
    assert L.ft2_protect_fused_gemm(P(0x1000), 12, P(0x2000), 12, None, P(0x3000), 16, 4, 16, 12, 0, 0, 0, 16,
                                    None, None, 0, None, None, 0, 0, 0, None, None, 0, None) == FT2_ERR_MISALIGNED
    # fused gemm CHECK without bounds
    assert L.ft2_protect_fused_gemm(P(0x1000), 16, P(0x2000), 16, None, P(0x3000), 16, 4, 16, 16, 1, 0, 0, 16,
                                    None, None, 1, None, None, 0, 0, 0, None, None, 0, None) == FT2_ERR_INVALID_ARG


def test_fused_gemm_ex_prefetch_hint_validation(L):
    from paper_conf_hpdc_sunzmg00y25_b200._lib import FT2_ERR_INVALID_ARG, FT2_ERR_MISALIGNED, FT2_ERR_UNSUPPORTED
    P = ctypes.c_void_p

    def ex(pf, nbytes, dtype=0, M=4):
        return L.ft2_protect_fused_gemm_ex(P(0x1000), 16, P(0x2000), 16, None, P(0x3000), 16, M, 16, 16, 0, dtype,
                                           0, 16, None, None, 0, None, None, 0, 0, 0, None, None, 0, pf, nbytes, None)
    assert ex(None, 16) == FT2_ERR_INVALID_ARG          # bytes without a pointer
    assert ex(P(0x4008), 16) == FT2_ERR_MISALIGNED      # pointer not 16-byte aligned
    assert ex(P(0x4000), 24) == FT2_ERR_MISALIGNED      # size not a multiple of 16
    assert ex(P(0x4000), 32, dtype=2) == FT2_ERR_UNSUPPORTED   # then the ft2_protect_fused_gemm checks
    assert ex(None, 0, dtype=2) == FT2_ERR_UNSUPPORTED


def test_host_kernel_wrappers_reject_mismatched_tensors():
    """the host-model wrappers check what the C ABI cannot see
    (dtypes, widths, shapes) before any launch."""
    import torch
    from paper_conf_hpdc_sunzmg00y25_b200 import ft2
    x = torch.zeros((4, 16), dtype=torch.bfloat16)
    y = torch.zeros((4, 16), dtype=torch.bfloat16)
    with pytest.raises(ValueError):
        ft2.host_norm(x, torch.ones(16, dtype=torch.float32), y)           # fp32 weight read as bf16
    with pytest.raises(ValueError):
        ft2.host_norm(x, torch.ones(8, dtype=torch.bfloat16), y)           # narrow weight
    with pytest.raises(ValueError):
        ft2.host_norm(x, torch.ones(16, dtype=torch.bfloat16), torch.zeros((2, 16), dtype=torch.bfloat16))
    with pytest.raises(ValueError):
        ft2.host_act(x, y, b=torch.zeros((4, 8), dtype=torch.bfloat16), act="silu_mul")   # narrow b
    with pytest.raises(ValueError):
        ft2.host_act(x, torch.zeros((4, 16), dtype=torch.float16))        # y dtype
