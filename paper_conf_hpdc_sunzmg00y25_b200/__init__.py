"""FT2 on B200: online range restriction of critical LLM layers (sm_100a).

Product package.  It never imports ``oracle/``; compute runs only in
``lib/libft2.so`` (built from ``csrc/`` for sm_100a).  Importing the package
loads the library and raises if it is missing -- there is no CPU fallback.
"""
from ._lib import load as _load

_load()

from . import ft2  # noqa: E402,F401
from .ft2 import (allreduce_protect, bounds_finalize, bounds_from_prefill, gemm_workspace_bytes,  # noqa: E402,F401
                  inject_faults, launch_count, make_fault_sites, make_workspace, prefill_fused_gemm, protect,
                  protect_fused_gemm, version, workspace_bytes, host_norm, host_act)

__all__ = ["bounds_from_prefill", "bounds_finalize", "protect", "protect_fused_gemm", "prefill_fused_gemm",
           "make_fault_sites", "inject_faults", "allreduce_protect", "make_workspace", "workspace_bytes",
           "gemm_workspace_bytes", "launch_count", "version", "host_norm", "host_act"]
