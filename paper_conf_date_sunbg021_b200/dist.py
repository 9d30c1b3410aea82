"""Multi-GPU drivers: one process per GPU, torch.distributed (NCCL) plumbing.

Two ways Algorithm 2 spreads over GPUs (DESIGN.md
"Multi-GPU"):

1. `run_batches_dp` -- the B independent batch TEDs of Alg. 2 l.1-4 go
   round-robin over the ranks (batch b on rank b mod G; "our batch method can
   stimulate the parallelism").  The only exchange is the real
   one of Alg. 2 l.5: an all-gather of the m winners per batch (int64), after
   which every rank runs the identical merge TED (l.6) on its own GPU.

2. `ShardedTed` -- one oversized batch (Alg. 1 on N rows) with K row-sharded
   over the ranks.  Per step t the exchange is: all-reduce(MAX) of the packed
   argmax key (8 bytes) and an all-gather of column s_t of K over the bands
   (4N bytes), which IS row s_t (K is bitwise symmetric) -- the pivot row the
   next deflation needs.  Each rank's rows are computed exactly as on one GPU
   (every row's reduction order depends on N only), so the selection is
   bit-identical to `bted_select` for any number of shards.

Every step of the method runs in libbted.so's kernels; this module only
moves buffers between them (the `comm` object) and owns no arithmetic.
"""
from __future__ import annotations

import math

import numpy as np
import torch

from . import _lib as L


# ---------------------------------------------------------------- comms
class TorchComm:
    """Collectives over torch.distributed (NCCL on GPUs, gloo in CPU tests)."""

    def __init__(self, group=None):
        import torch.distributed as dist
        self.dist = dist
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)

    def allreduce_max_(self, t: torch.Tensor):
        self.dist.all_reduce(t, op=self.dist.ReduceOp.MAX, group=self.group)

    def allgather_(self, out: torch.Tensor, inp: torch.Tensor):
        self.dist.all_gather_into_tensor(out, inp, group=self.group)


def band(N: int, P: int, r: int):
    """Rows [row0, row1) of shard r: equal bands of ceil(N/P) rows (last may be short)."""
    B = math.ceil(N / P)
    return min(N, r * B), min(N, (r + 1) * B), B


# ------------------------------------------------------- 1. batch round-robin
def run_batches_dp(pool_ctx: int, M: int, m: int, mu: float, B: int, comm, device: torch.device):
    """Alg. 2 over `comm.world` ranks.  Returns (X pool indices, per-rank winners)."""
    G, r = comm.world, comm.rank
    nb_max = math.ceil(B / G)
    nb_local = len(range(r, B, G))
    win = torch.full((nb_max * m,), -1, dtype=torch.int64, device=device)
    if nb_local:
        L.bted_batch_teds(pool_ctx, M, m, mu, r, G, win.data_ptr(), winners_on_device=True)
    allw = torch.empty((G * nb_max * m,), dtype=torch.int64, device=device)
    comm.allgather_(allw, win)                       # Alg. 2 l.5 exchange (padding = -1)
    torch.cuda.current_stream(device).synchronize()
    sel = L.bted_merge(pool_ctx, allw.data_ptr(), allw.numel(), m, mu, winners_on_device=True)
    return sel, win


# ------------------------------------------------------- 2. row-sharded TED
class ShardedTed:
    """TED on N rows with this rank's band of K (rows [row0, row1))."""

    def __init__(self, X, N: int, d: int, gamma: float, comm, device: torch.device, stream: torch.cuda.Stream,
                 kernel: int = L.BTED_KERNEL_RBF):
        self.N, self.d, self.comm, self.device, self.stream = int(N), int(d), comm, device, stream
        self.row0, self.row1, self.bandB = band(self.N, comm.world, comm.rank)
        p = L.default_params(gamma=gamma, device=device.index, stream=stream.cuda_stream,
                             x_on_device=1 if isinstance(X, int) else 0)
        self.ctx = L.bted_shard_create(X, N, d, kernel, self.row0, self.row1, p)
        self.ld = L.bted_shard_ld(self.ctx)
        width = max(self.ld, comm.world * self.bandB)
        with torch.cuda.stream(stream):
            self.pivot = torch.zeros(width, dtype=torch.float32, device=device)
            self.col = torch.zeros(self.bandB, dtype=torch.float32, device=device)

    def select(self, m: int, mu: float):
        if not (1 <= m <= self.N):
            raise ValueError("need 1 <= m <= N")
        P = self.comm.world
        with torch.cuda.stream(self.stream):
            keys = torch.zeros(m, dtype=torch.int64, device=self.device)
            kp = keys.data_ptr()
            L.bted_shard_gram(self.ctx, mu, kp)                   # l.1 + first l.3 on the band
            self.comm.allreduce_max_(keys[0:1])                   # global argmax s_1
            gathered = self.pivot[: P * self.bandB]
            for t in range(1, m):
                L.bted_shard_pivot_column(self.ctx, t - 1, kp, self.col.data_ptr())
                self.comm.allgather_(gathered, self.col)          # column s_t == row s_t
                L.bted_shard_step(self.ctx, t, mu, self.pivot.data_ptr(), kp)   # l.5 + next l.3
                self.comm.allreduce_max_(keys[t:t + 1])
            host = keys.cpu().numpy().view(np.uint64)
        L.bted_shard_check(self.ctx)
        return L.decode_keys(host)

    def close(self):
        if getattr(self, "ctx", None):
            L.bted_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ------------------------------------------------ loopback (P shards, 1 GPU)
def sharded_select_loopback(X: np.ndarray, gamma: float, P: int, m: int, mu: float, device: torch.device,
                            stream: torch.cuda.Stream, kernel: int = L.BTED_KERNEL_RBF):
    """The ShardedTed exchange with P logical shards on ONE GPU; the two
    collectives are emulated by device copies / a max.  Exercises the sharded
    control flow and its bit-identity without a second GPU."""
    N, d = X.shape
    ctxs, bands = [], []
    p = L.default_params(gamma=gamma, device=device.index, stream=stream.cuda_stream)
    try:
        for r in range(P):
            r0, r1, Bw = band(N, P, r)
            ctxs.append(L.bted_shard_create(X, N, d, kernel, r0, r1, p))
            bands.append((r0, r1))
        ld = L.bted_shard_ld(ctxs[0])
        with torch.cuda.stream(stream):
            keys = torch.zeros((P, m), dtype=torch.int64, device=device)
            pivot = torch.zeros(max(ld, P * Bw), dtype=torch.float32, device=device)
            cols = torch.zeros((P, Bw), dtype=torch.float32, device=device)
            for r in range(P):
                L.bted_shard_gram(ctxs[r], mu, keys[r].data_ptr())
            keys[:, 0] = keys[:, 0].max()
            for t in range(1, m):
                for r in range(P):
                    L.bted_shard_pivot_column(ctxs[r], t - 1, keys[r].data_ptr(), cols[r].data_ptr())
                pivot[: P * Bw].copy_(cols.reshape(-1))
                for r in range(P):
                    L.bted_shard_step(ctxs[r], t, mu, pivot.data_ptr(), keys[r].data_ptr())
                keys[:, t] = keys[:, t].max()
            host = keys[0].cpu().numpy().view(np.uint64)
        for c in ctxs:
            L.bted_shard_check(c)
        return L.decode_keys(host)
    finally:
        for c in ctxs:
            L.bted_destroy(c)
