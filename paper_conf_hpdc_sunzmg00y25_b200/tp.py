"""Tensor-parallel bounds combine.

PAPER.md's FT2 is single-GPU (L280).  When a critical layer is column-parallel
(V_PROJ, UP_PROJ in Megatron TP), every rank holds a column shard of the
prefill output.  The per-sequence bounds of the full output are the min/max
over shards, which is exact and associative:

    1. each rank: ft2_bounds_from_prefill(shard, finalize=0, keys_out=keys)
       keys[s] = (0xFFFF - key(lo_raw), key(hi_raw)), -1 = no finite value
    2. all ranks: all_reduce(keys, MAX)            (one int32 [L_col, B, 2] call)
    3. each rank: ft2_bounds_finalize(keys) -> bf16 bounds (x2 widening, R3)

Scaling commutes with min/max (the widening is monotone), so the result is
bit-identical to single-GPU bounds.  Row-parallel layers (OUT/O_PROJ,
DOWN_PROJ/FC2) are checked after their own sum all-reduce (reading A17): every
rank then holds the full output and computes identical bounds locally.

The all-reduce is NCCL over NVLink/NVSwitch on GPUs; the same code runs on
gloo for the CPU tests.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

KEY_NONE = -1


def allreduce_bounds_keys(keys: torch.Tensor, group=None) -> torch.Tensor:
    """Element-wise MAX all-reduce of int32 keys [..., 2] in the ABI encoding, in place."""
    if keys.dtype != torch.int32 or keys.shape[-1] != 2:
        raise ValueError("keys must be int32 [..., 2] in the ft2_bounds_from_prefill encoding")
    dist.all_reduce(keys, op=dist.ReduceOp.MAX, group=group)
    return keys


def decode_keys(keys: torch.Tensor):
    """ABI-encoded keys -> (key(lo_raw), key(hi_raw)) int tensors, -1 where a sequence has no finite value."""
    lo = torch.where(keys[..., 0] >= 0, 0xFFFF - keys[..., 0], torch.full_like(keys[..., 0], KEY_NONE))
    hi = keys[..., 1]
    return lo, hi


def tp_bounds_from_prefill(y_shard: torch.Tensor, bounds_out: torch.Tensor, workspace: torch.Tensor,
                           seq_offsets=None, num_seqs=None, scale: float = 2.0, group=None,
                           keys: torch.Tensor = None) -> torch.Tensor:
    """Bounds of a column-parallel layer's full prefill output from this rank's shard.

    Runs the bounds kernel (keys only), one MAX all-reduce, then the finalize
    kernel.  bounds_out: bf16 [S, 2].  Returns the all-reduced keys."""
    from . import ft2 as F2

    S = num_seqs if num_seqs is not None else (1 if seq_offsets is None else seq_offsets.numel() - 1)
    if keys is None:
        keys = torch.empty((S, 2), dtype=torch.int32, device=y_shard.device)
    F2.bounds_from_prefill(y_shard, None, workspace, seq_offsets=seq_offsets, num_seqs=S, scale=scale,
                           finalize=False, keys_out=keys)
    allreduce_bounds_keys(keys, group=group)
    F2.bounds_finalize(keys, bounds_out, scale=scale)
    return keys


def column_shard(n: int, world: int, rank: int):
    """[begin, end) output columns of `rank` for an n-wide column-parallel layer."""
    per = (n + world - 1) // world
    b = min(n, rank * per)
    return b, min(n, b + per)


class RowParallelCheck:
    """A row-parallel critical layer's sum all-reduce fused with FT2's check
    (ft2_allreduce_protect, reading A17).

    Owns this rank's double-buffered partial outputs [2, rows, n], its flag
    array [P] and its (epoch, done, status) words; exchanges CUDA IPC handles
    once over `group` (any backend: the handles are host bytes) and maps every
    peer's buffers.  Call i writes its GEMM partial into partial(i) and then
    calls __call__(i, ...); consecutive calls must alternate i's parity."""

    def __init__(self, rows: int, n: int, dtype=torch.bfloat16, group=None, device=None):
        from . import ft2 as F2
        self.F2 = F2
        self.P = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        dev = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        self.rows, self.n = rows, n
        self.partials = torch.zeros((2, rows, n), dtype=dtype, device=dev)
        self.flags = torch.zeros(self.P, dtype=torch.int32, device=dev)
        self.words = torch.zeros(3, dtype=torch.int32, device=dev)
        mine = (F2.ipc_get_handle(self.partials), F2.ipc_get_handle(self.flags))
        allh = [None] * self.P
        dist.all_gather_object(allh, mine, group=group)
        self._opened = []
        pptr, fptr = [], []
        elt = self.partials.element_size()
        for t, ((hp, op), (hf, of)) in enumerate(allh):
            if t == self.rank:
                bp, bf = self.partials.data_ptr(), self.flags.data_ptr()
            else:
                basep = F2.ipc_open_handle(hp)
                basef = F2.ipc_open_handle(hf) if hf != hp else basep
                self._opened += [basep] + ([basef] if basef != basep else [])
                bp, bf = basep + op, basef + of
            pptr.append((bp, bp + rows * n * elt))
            fptr.append(bf)
        self.partial_ptrs = [[p[b] for p in pptr] for b in (0, 1)]   # host ints, passed by value
        self.flag_ptrs = list(fptr)
        dist.barrier(group=group)   # every rank mapped everything before any call

    def partial(self, i: int) -> torch.Tensor:
        return self.partials[i & 1]

    def __call__(self, i: int, y: torch.Tensor, bias=None, mode=1, bounds=None, row_to_seq=None, num_seqs=None,
                 corrected_count=None, sites=None, n_sites=None, cur_layer=0, cur_step=0, base_row=None):
        self.F2.allreduce_protect(self.partial_ptrs[i & 1], self.n, self.P, self.rank, self.flag_ptrs, self.words, y,
                                  bias=bias, mode=mode, bounds=bounds, row_to_seq=row_to_seq, num_seqs=num_seqs,
                                  corrected_count=corrected_count, sites=sites, n_sites=n_sites,
                                  cur_layer=cur_layer, cur_step=cur_step, base_row=base_row)

    def status(self) -> int:
        return int(self.words[2].item())

    def close(self):
        for b in self._opened:
            self.F2.ipc_close(b)
        self._opened = []
