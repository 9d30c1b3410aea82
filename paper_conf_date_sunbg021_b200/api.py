"""Object wrapper over the C ABI (ownership only; no arithmetic)."""
from __future__ import annotations

import numpy as np

from . import _lib as L


class CandidateSet:
    """A candidate set V / pool on one GPU (bted_create ... bted_destroy).

    X: host np.float32 [N, d], or a CUDA torch tensor (adopted, must outlive
    this object).  `select` = TED (Alg. 1), `run_batches` = BTED (Alg. 2).
    num_devices > 1: one ctx drives GPUs [device, device + num_devices) --
    run_batches round-robins the batches, select tile-shards the candidate set
    (flags BTED_FLAG_LOOPBACK: logical devices on one GPU; BTED_FLAG_NCCL:
    exchange through NCCL instead of peer memory).
    """

    def __init__(self, X, gamma: float, *, kernel: int = L.BTED_KERNEL_RBF, num_batches: int = 1,
                 seed: int = 0, device: int = -1, flags: int = 0, stream: int = 0, num_devices: int = 1,
                 norm_mode: int = 0):
        self._x_ref = X
        on_dev = hasattr(X, "is_cuda") and X.is_cuda
        if on_dev:
            if X.dtype.__repr__() != "torch.float32" or not X.is_contiguous():
                raise ValueError("device X must be a contiguous float32 CUDA tensor")
            N, d = X.shape
            ptr = X.data_ptr()
            device = X.device.index if device < 0 else device
        else:
            X = np.ascontiguousarray(X, dtype=np.float32)
            N, d = X.shape
            ptr = X
        self.N, self.d, self.num_batches = int(N), int(d), int(num_batches)
        p = L.default_params(gamma=gamma, device=device, num_batches=num_batches, seed=seed,
                             x_on_device=1 if on_dev else 0, flags=flags, stream=stream,
                             num_devices=num_devices, norm_mode=norm_mode)
        self.ctx = L.bted_create(ptr, N, d, kernel, p)

    def update(self, X, on_device: bool = False):
        """Replace the features (same N x d): a host array is shape-checked and
        converted to C-contiguous fp32; a CUDA tensor is copied D2D."""
        if hasattr(X, "is_cuda") and X.is_cuda:
            if tuple(X.shape) != (self.N, self.d) or str(X.dtype) != "torch.float32" or not X.is_contiguous():
                raise ValueError("update: need a contiguous float32 CUDA tensor of shape (N, d)")
            self._x_update_ref = X
            return L.bted_update(self.ctx, X.data_ptr(), x_on_device=True)
        return L.bted_update(self.ctx, X, shape=(self.N, self.d))

    def select(self, m: int, mu: float):
        return L.bted_select(self.ctx, m, mu)

    def run_batches(self, M: int, m: int, mu: float, want_batches: bool = True):
        return L.bted_run_batches(self.ctx, M, m, mu, self.num_batches, want_batches)

    def batch_teds(self, M: int, m: int, mu: float, b_begin: int, b_step: int, out, on_device: bool = False):
        return L.bted_batch_teds(self.ctx, M, m, mu, b_begin, b_step, out, on_device)

    def merge(self, winners, n: int, m: int, mu: float, on_device: bool = False):
        return L.bted_merge(self.ctx, winners, n, m, mu, on_device)

    def debug_K(self, rows: int, which: int = 0) -> np.ndarray:
        ld = (self.N + 31) // 32 * 32 if which == 0 else None
        return L.bted_debug_copy_K(self.ctx, which, rows, ld)

    def close(self):
        if getattr(self, "ctx", None):
            L.bted_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()
