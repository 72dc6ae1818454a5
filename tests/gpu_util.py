"""Helpers for GPU parity tests: move column-major numpy matrices to/from torch CUDA."""
import numpy as np
import torch

import rgsqr_inputs as gi

TORCH_DT = {"fp16": torch.float16, "bf16": torch.bfloat16, "fp32": torch.float32}


def to_dev(a_stored: np.ndarray, storage: str) -> torch.Tensor:
    """Stored column-major m x n numpy matrix -> CUDA tensor At (n, m) (A[i,j] = At[j,i])."""
    at = np.ascontiguousarray(a_stored.T)
    if storage == "bf16":
        return torch.from_numpy(at.view(np.int16)).view(torch.bfloat16).cuda()
    return torch.from_numpy(at).cuda()


def from_dev(at: torch.Tensor) -> np.ndarray:
    """CUDA tensor At (n, m) -> float64 numpy m x n (exact widening)."""
    return at.detach().to(torch.float64).cpu().numpy().T.copy(order="F")


def stored(a64: np.ndarray, storage: str) -> np.ndarray:
    return gi.to_storage(a64, storage)
