"""Device-buffer helpers for the GPU tests (torch = device memory only).

While a MasterKernel is resident it holds every warp of the GPU, so no torch
KERNEL may run between pagoda init and shutdown (copies are fine): every
buffer here is allocated and filled with copies, never with fill kernels,
and tests allocate before they start Pagoda.
"""
import numpy as np
import torch


class Dev:
    """Keeps device tensors alive; hands out raw pointers."""

    def __init__(self):
        self.keep = []

    def put(self, a: np.ndarray) -> torch.Tensor:
        a = np.ascontiguousarray(a)
        t = torch.empty(a.nbytes, dtype=torch.uint8, device="cuda")
        t.copy_(torch.from_numpy(a.view(np.uint8).reshape(-1)))
        self.keep.append(t)
        return t

    def zeros(self, nbytes: int) -> torch.Tensor:
        return self.put(np.zeros(nbytes, np.uint8))

    @staticmethod
    def get(t: torch.Tensor, dtype, shape=None) -> np.ndarray:
        a = t.cpu().numpy().view(dtype)
        return a.reshape(shape) if shape is not None else a


def ptr(t: torch.Tensor) -> int:
    return t.data_ptr()
