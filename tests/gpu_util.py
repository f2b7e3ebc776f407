"""Helpers shared by the GPU parity tests (host <-> device bit patterns)."""
import numpy as np
import torch


def dev(a: np.ndarray) -> torch.Tensor:
    """uint16 bf16 bits (numpy) -> CUDA bfloat16 tensor (same shape)."""
    a = np.ascontiguousarray(a, dtype=np.uint16)
    return torch.from_numpy(a.view(np.int16)).view(torch.bfloat16).cuda()


def host(t: torch.Tensor) -> np.ndarray:
    """CUDA/CPU bfloat16 tensor -> uint16 bf16 bits (numpy)."""
    return t.detach().contiguous().cpu().view(torch.int16).numpy().view(np.uint16)


def dev_i32(a) -> torch.Tensor:
    return torch.as_tensor(np.asarray(a, dtype=np.int32)).cuda()


def sites_to_host(sites_u8: torch.Tensor, dtype) -> np.ndarray:
    return sites_u8.cpu().numpy().view(dtype)


def sites_to_dev(sites_np: np.ndarray) -> torch.Tensor:
    return torch.from_numpy(np.ascontiguousarray(sites_np).view(np.uint8).copy()).cuda()
