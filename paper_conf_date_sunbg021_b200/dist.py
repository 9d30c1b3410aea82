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
   `norm_mode="literal"` is the north_star's literal exchange instead: every
   rank sums its band's part of each COLUMN norm (Alg. 1 l.3),
   an all-reduce(SUM) of those N floats gives ||K_v||^2, and each rank scores
   its own indices from it (then the same argmax all-reduce).  Same band
   values; the scores differ from the symmetric mode only in rounding order.

3. `ShardedImplicitTed` -- the same oversized batch on the default implicit
   engine: the read-only packed Gram tiles are split over the ranks (tile k on
   rank k mod P), everything else is replicated; per step one all-reduce(SUM)
   of the partial q = K l vectors.

Every step of the method runs in libbted.so's kernels (the `LibShard` /
`LibPool` backends below); this module only moves buffers between them
through the `comm` object and owns no arithmetic.  The backends are
injectable so the exchange protocol itself is covered by CPU (gloo) tests.
"""
from __future__ import annotations

import contextlib
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

    def allreduce_sum_(self, t: torch.Tensor):
        self.dist.all_reduce(t, op=self.dist.ReduceOp.SUM, group=self.group)

    def allgather_(self, out: torch.Tensor, inp: torch.Tensor):
        self.dist.all_gather_into_tensor(out, inp, group=self.group)


def band(N: int, P: int, r: int):
    """Rows [row0, row1) of shard r: equal bands of ceil(N/P) rows (last may be short)."""
    B = math.ceil(N / P)
    return min(N, r * B), min(N, (r + 1) * B), B


def _stream_ctx(stream):
    return torch.cuda.stream(stream) if stream is not None else contextlib.nullcontext()


# ------------------------------------------------------- 1. batch round-robin
class LibPool:
    """Backend of run_batches_dp: a pool ctx of libbted.so."""

    def __init__(self, ctx: int):
        self.ctx = ctx

    def batch_teds(self, M, m, mu, b_begin, b_step, out: torch.Tensor):
        if out.is_cuda:
            # `out` was written (e.g. filled with -1) on torch's current stream; the
            # library writes the winners on the ctx's own stream: order the two
            torch.cuda.current_stream(out.device).synchronize()
        L.bted_batch_teds(self.ctx, M, m, mu, b_begin, b_step, out.data_ptr(), winners_on_device=out.is_cuda)

    def merge(self, winners: torch.Tensor, m, mu):
        if winners.is_cuda:
            torch.cuda.current_stream(winners.device).synchronize()
            return L.bted_merge(self.ctx, winners.data_ptr(), winners.numel(), m, mu, winners_on_device=True)
        return L.bted_merge(self.ctx, winners.numpy(), winners.numel(), m, mu)


def run_batches_dp(pool, M: int, m: int, mu: float, B: int, comm, device: torch.device):
    """Alg. 2 over `comm.world` ranks.  pool: LibPool or a pool ctx handle.
    Returns (X pool indices, this rank's winners with -1 padding)."""
    if isinstance(pool, int):
        pool = LibPool(pool)
    G, r = comm.world, comm.rank
    nb_max = math.ceil(B / G)
    nb_local = len(range(r, B, G))
    win = torch.full((nb_max * m,), -1, dtype=torch.int64, device=device)
    if nb_local:
        pool.batch_teds(M, m, mu, r, G, win)         # l.1-4 for b = r, r+G, ...
    allw = torch.empty((G * nb_max * m,), dtype=torch.int64, device=device)
    comm.allgather_(allw, win)                       # l.5 exchange (padding = -1)
    return pool.merge(allw, m, mu), win              # l.5 union + l.6 merge TED


# ------------------------------------------------------- 2. row-sharded TED
class LibShard:
    """Backend of ShardedTed: a shard ctx of libbted.so (rows [row0, row1))."""

    def __init__(self, X, N, d, gamma, row0, row1, device: torch.device, stream, kernel=L.BTED_KERNEL_RBF):
        on_dev = isinstance(X, int)
        p = L.default_params(gamma=gamma, device=device.index, stream=stream.cuda_stream,
                             x_on_device=1 if on_dev else 0)
        self.ctx = L.bted_shard_create(X, N, d, kernel, row0, row1, p)
        self.ld = L.bted_shard_ld(self.ctx)

    def gram(self, mu, keys: torch.Tensor):
        L.bted_shard_gram(self.ctx, mu, keys.data_ptr())

    def pivot_column(self, t, keys: torch.Tensor, col: torch.Tensor):
        L.bted_shard_pivot_column(self.ctx, t, keys.data_ptr(), col.data_ptr())

    def step(self, t, mu, pivot: torch.Tensor, keys: torch.Tensor):
        L.bted_shard_step(self.ctx, t, mu, pivot.data_ptr(), keys.data_ptr())

    def nearties(self, m, keys: torch.Tensor, cand: torch.Tensor, ncand: torch.Tensor):
        L.bted_shard_nearties(self.ctx, m, keys.data_ptr(), cand.data_ptr(), ncand.data_ptr())

    def refine(self, m, mu, keys: torch.Tensor, cand_all: np.ndarray, ncand_all: np.ndarray, nranks: int):
        return L.bted_shard_refine(self.ctx, m, mu, keys.data_ptr(), cand_all, ncand_all, nranks)

    def colnorm(self, t, mu, pivot, keys, colnorm: torch.Tensor):
        L.bted_shard_colnorm(self.ctx, t, mu, pivot.data_ptr() if pivot is not None else None,
                             keys.data_ptr() if keys is not None else None, colnorm.data_ptr())

    def scores(self, t, mu, colnorm: torch.Tensor, keys: torch.Tensor):
        L.bted_shard_scores(self.ctx, t, mu, colnorm.data_ptr(), keys.data_ptr())

    def check(self):
        L.bted_shard_check(self.ctx)

    def close(self):
        if self.ctx:
            L.bted_destroy(self.ctx)
            self.ctx = None


class ShardedTed:
    """TED (Alg. 1) on N rows with this rank's band of K.  `backend` runs the
    band's kernels (LibShard on a GPU); `comm` does the two per-step exchanges.
    With `graph=True` (GPU, a CUDA stream given) the whole m-step loop --
    kernels AND the NCCL collectives -- is captured once per (m, mu) into a
    CUDA graph and replayed: no per-step host work."""

    def __init__(self, backend, N: int, comm, device: torch.device, stream=None, graph: bool = False,
                 norm_mode: str = "symmetric"):
        if norm_mode not in ("symmetric", "literal"):
            raise ValueError("norm_mode must be 'symmetric' or 'literal'")
        self.norm_mode = norm_mode
        self.be, self.N, self.comm, self.device, self.stream = backend, int(N), comm, device, stream
        self.row0, self.row1, self.bandB = band(self.N, comm.world, comm.rank)
        width = max(getattr(backend, "ld", self.N), comm.world * self.bandB)
        self.graph = bool(graph) and stream is not None
        self._graphs = {}
        with _stream_ctx(stream):
            self.pivot = torch.zeros(width, dtype=torch.float32, device=device)
            self.col = torch.zeros(self.bandB, dtype=torch.float32, device=device)
            if norm_mode == "literal":
                self.cn = torch.zeros(width, dtype=torch.float32, device=device)
                self.scratch = torch.zeros(1, dtype=torch.int64, device=device)

    def _loop_literal(self, keys: torch.Tensor, m: int, mu: float, preset=None):
        P = self.comm.world
        keys.zero_()
        if preset is not None:                                    # K4: forced picks win every max
            keys[: len(preset)].copy_(torch.from_numpy(preset.view(np.int64)))
        self.be.gram(mu, self.scratch)                            # l.1 on the band
        self.be.colnorm(0, mu, None, None, self.cn)               # band part of every column norm
        self.comm.allreduce_sum_(self.cn)                         # ||K_v||^2 (N floats)
        self.be.scores(0, mu, self.cn, keys)                      # l.3 for the band's own v
        self.comm.allreduce_max_(keys[0:1])                       # s_1
        gathered = self.pivot[: P * self.bandB]
        for t in range(1, m):
            self.be.pivot_column(t - 1, keys, self.col)
            self.comm.allgather_(gathered, self.col)              # pivot row s_t (4N B)
            self.be.colnorm(t, mu, self.pivot, keys, self.cn)     # l.5 on the band + column partials
            self.comm.allreduce_sum_(self.cn)
            self.be.scores(t, mu, self.cn, keys)
            self.comm.allreduce_max_(keys[t:t + 1])               # s_{t+1}

    def _loop(self, keys: torch.Tensor, m: int, mu: float, preset=None):
        if self.norm_mode == "literal":
            return self._loop_literal(keys, m, mu, preset)
        P = self.comm.world
        keys.zero_()
        if preset is not None:                                    # K4: forced picks win every max
            keys[: len(preset)].copy_(torch.from_numpy(preset.view(np.int64)))
        self.be.gram(mu, keys)                                    # l.1 + first l.3 on the band
        self.comm.allreduce_max_(keys[0:1])                       # global argmax s_1 (8 B)
        gathered = self.pivot[: P * self.bandB]
        for t in range(1, m):
            self.be.pivot_column(t - 1, keys, self.col)           # K[band, s_t]
            self.comm.allgather_(gathered, self.col)              # column s_t == row s_t (4N B)
            self.be.step(t, mu, self.pivot, keys)                 # l.5 + next l.3 on the band
            self.comm.allreduce_max_(keys[t:t + 1])               # s_{t+1}

    def select(self, m: int, mu: float):
        if not (1 <= m <= self.N):
            raise ValueError("need 1 <= m <= N")
        with _stream_ctx(self.stream):
            if self.graph:
                gk = (int(m), float(mu))
                if gk not in self._graphs:
                    keys = torch.zeros(m, dtype=torch.int64, device=self.device)
                    self._loop(keys, m, mu)                       # eager once: allocations, NCCL init
                    g = torch.cuda.CUDAGraph()
                    with torch.cuda.graph(g, stream=self.stream):
                        self._loop(keys, m, mu)
                    self._graphs[gk] = (g, keys)
                g, keys = self._graphs[gk]
                g.replay()
            else:
                keys = torch.zeros(m, dtype=torch.int64, device=self.device)
                self._loop(keys, m, mu)
            if hasattr(self.be, "nearties"):
                for _ in range(m):                                # K4 (identical decision on every rank)
                    forced = self._k4(keys, m, mu)
                    if len(forced) == 0:
                        break
                    keys = torch.zeros(m, dtype=torch.int64, device=self.device)
                    self._loop(keys, m, mu, preset=forced)
            host = keys.cpu().numpy().view(np.uint64)
        self.be.check()
        return L.decode_keys(host)

    def _k4(self, keys: torch.Tensor, m: int, mu: float):
        P = self.comm.world
        cand = torch.zeros((m, 32), dtype=torch.int32, device=self.device)
        ncand = torch.zeros(m, dtype=torch.int32, device=self.device)
        self.be.nearties(m, keys, cand, ncand)
        cand_all = torch.empty((P * m, 32), dtype=torch.int32, device=self.device)
        ncand_all = torch.empty(P * m, dtype=torch.int32, device=self.device)
        self.comm.allgather_(cand_all, cand)
        self.comm.allgather_(ncand_all, ncand)
        return self.be.refine(m, mu, keys, cand_all.cpu().numpy().view(np.uint32), ncand_all.cpu().numpy(), P)


# ------------------------------------------- 3. tile-sharded implicit TED
class LibIShard:
    """Backend of ShardedImplicitTed: a tile-shard ctx of libbted.so (Gram tiles k = rank mod P)."""

    def __init__(self, X, N, d, gamma, rank, nranks, device: torch.device, stream, kernel=L.BTED_KERNEL_RBF):
        on_dev = isinstance(X, int)
        p = L.default_params(gamma=gamma, device=device.index, stream=stream.cuda_stream,
                             x_on_device=1 if on_dev else 0)
        self.ctx = L.bted_ishard_create(X, N, d, kernel, rank, nranks, p)
        self.qlen = L.bted_ishard_qlen(self.ctx)

    def head(self, m, mu, q: torch.Tensor):
        L.bted_ishard_head(self.ctx, m, mu, q.data_ptr())

    def step(self, t, mu, keys: torch.Tensor, q: torch.Tensor):
        L.bted_ishard_step(self.ctx, t, mu, keys.data_ptr(), q.data_ptr())

    def fin(self, t, mu, q: torch.Tensor, keys: torch.Tensor):
        L.bted_ishard_fin(self.ctx, t, mu, q.data_ptr(), keys.data_ptr())

    def refine(self, m, mu, keys: torch.Tensor):
        return L.bted_ishard_refine(self.ctx, m, mu, keys.data_ptr())

    def check(self):
        L.bted_shard_check(self.ctx)

    def close(self):
        if self.ctx:
            L.bted_destroy(self.ctx)
            self.ctx = None


class ShardedImplicitTed:
    """TED (Alg. 1) on N points with the implicit engine's packed Gram tiles
    split over the ranks (tile k on rank k mod P).  Per step ONE collective:
    all-reduce(SUM) of the ranks' partial q = K l (qlen fp64); every rank then
    computes the same scores and argmax from its replicated O(N m) state.
    Per-rank HBM traffic per step ~ 2 N^2 / P bytes (vs 8 N^2 / P for the
    dense-band ShardedTed).  `graph=True` captures the m-step loop, kernels
    and NCCL collectives, into one CUDA graph per (m, mu)."""

    def __init__(self, backend, N: int, comm, device: torch.device, stream=None, graph: bool = False):
        self.be, self.N, self.comm, self.device, self.stream = backend, int(N), comm, device, stream
        self.graph = bool(graph) and stream is not None
        self._graphs = {}
        with _stream_ctx(stream):
            self.q = torch.zeros(backend.qlen, dtype=torch.float64, device=device)

    def _loop(self, keys: torch.Tensor, m: int, mu: float, preset=None):
        keys.zero_()
        if preset is not None:                       # K4: forced picks (flagged keys win every max)
            keys[: len(preset)].copy_(torch.from_numpy(preset.view(np.int64)))
        self.be.head(m, mu, self.q)                  # l.1 + this rank's part of ||K_:v||^2
        self.comm.allreduce_sum_(self.q)
        self.be.fin(0, mu, self.q, keys)             # l.3: s_1 (identical on every rank)
        for t in range(1, m):
            self.be.step(t, mu, keys, self.q)        # l.5 implicitly: l_t, this rank's part of K l_t
            self.comm.allreduce_sum_(self.q)
            self.be.fin(t, mu, self.q, keys)         # next l.3: s_{t+1}

    def select(self, m: int, mu: float):
        if not (1 <= m <= self.N):
            raise ValueError("need 1 <= m <= N")
        with _stream_ctx(self.stream):
            if self.graph:
                gk = (int(m), float(mu))
                if gk not in self._graphs:
                    keys = torch.zeros(m, dtype=torch.int64, device=self.device)
                    self._loop(keys, m, mu)          # eager once: allocations, NCCL init
                    g = torch.cuda.CUDAGraph()
                    with torch.cuda.graph(g, stream=self.stream):
                        self._loop(keys, m, mu)
                    self._graphs[gk] = (g, keys)
                g, keys = self._graphs[gk]
                g.replay()
            else:
                keys = torch.zeros(m, dtype=torch.int64, device=self.device)
                self._loop(keys, m, mu)
            # K4: re-score near ties exactly; a changed pick re-runs the loop with the prefix forced
            # (identical decision on every rank, so the collectives stay matched)
            for _ in range(m):
                forced = self.be.refine(m, mu, keys) if hasattr(self.be, "refine") else []
                if len(forced) == 0:
                    break
                keys = torch.zeros(m, dtype=torch.int64, device=self.device)
                self._loop(keys, m, mu, preset=forced)
            host = keys.cpu().numpy().view(np.uint64)
        self.be.check()
        return L.decode_keys(host)


def isharded_select_loopback(X: np.ndarray, gamma: float, P: int, m: int, mu: float, device: torch.device,
                             stream: torch.cuda.Stream, kernel: int = L.BTED_KERNEL_RBF, stats: dict | None = None):
    """ShardedImplicitTed with P logical tile shards on ONE GPU; the all-reduce
    is a sum of the shards' partial q in rank order."""
    N, d = X.shape
    shards = []
    try:
        for r in range(P):
            shards.append(LibIShard(X, N, d, gamma, r, P, device, stream, kernel))
        with torch.cuda.stream(stream):
            keys = torch.zeros((P, m), dtype=torch.int64, device=device)
            qs = torch.zeros((P, shards[0].qlen), dtype=torch.float64, device=device)

            def allreduce():
                tot = qs[0].clone()
                for r in range(1, P):
                    tot += qs[r]
                qs.copy_(tot.expand_as(qs))

            def loop(preset=None):
                keys.zero_()
                if preset is not None:
                    keys[:, : len(preset)] = torch.from_numpy(preset.view(np.int64)).to(device)
                for r in range(P):
                    shards[r].head(m, mu, qs[r])
                allreduce()
                for r in range(P):
                    shards[r].fin(0, mu, qs[r], keys[r])
                for t in range(1, m):
                    for r in range(P):
                        shards[r].step(t, mu, keys[r], qs[r])
                    allreduce()
                    for r in range(P):
                        shards[r].fin(t, mu, qs[r], keys[r])

            loop()
            for _ in range(m):                                   # K4, as ShardedImplicitTed.select
                forced = [shards[r].refine(m, mu, keys[r]) for r in range(P)]
                assert all(np.array_equal(f, forced[0]) for f in forced), "shards disagree on K4"
                if len(forced[0]) == 0:
                    break
                loop(forced[0])
            host = keys.cpu().numpy().view(np.uint64)
        for s in shards:
            s.check()
        assert all((host[r] == host[0]).all() for r in range(P)), "shards disagree"
        if stats is not None:
            stats.update(L.bted_get_stats(shards[0].ctx))
        return L.decode_keys(host[0])
    finally:
        for s in shards:
            s.close()


# ------------------------------------------------ loopback (P shards, 1 GPU)
def sharded_select_loopback(X: np.ndarray, gamma: float, P: int, m: int, mu: float, device: torch.device,
                            stream: torch.cuda.Stream, kernel: int = L.BTED_KERNEL_RBF,
                            norm_mode: str = "symmetric", stats: dict | None = None):
    """The ShardedTed exchange with P logical shards on ONE GPU; the
    collectives are emulated by a device copy, a max and (literal norm mode)
    a sum over the shards in rank order.  Exercises the sharded kernels and
    their bit-identity without a second GPU."""
    N, d = X.shape
    literal = norm_mode == "literal"
    shards = []
    try:
        for r in range(P):
            r0, r1, Bw = band(N, P, r)
            shards.append(LibShard(X, N, d, gamma, r0, r1, device, stream, kernel))
        ld = shards[0].ld
        W = max(ld, P * Bw)
        with torch.cuda.stream(stream):
            keys = torch.zeros((P, m), dtype=torch.int64, device=device)
            pivot = torch.zeros(W, dtype=torch.float32, device=device)
            cols = torch.zeros((P, Bw), dtype=torch.float32, device=device)
            cn = torch.zeros((P, W), dtype=torch.float32, device=device)
            scratch = torch.zeros((P, 1), dtype=torch.int64, device=device)

            def scores(t):
                tot = cn[0].clone()
                for r in range(1, P):
                    tot += cn[r]
                for r in range(P):
                    shards[r].scores(t, mu, tot, keys[r])

            def rerun(preset=None):
                keys.zero_()
                if preset is not None:
                    keys[:, : len(preset)] = torch.from_numpy(preset.view(np.int64)).to(device)
                for r in range(P):
                    if literal:
                        shards[r].gram(mu, scratch[r])
                        shards[r].colnorm(0, mu, None, None, cn[r])
                    else:
                        shards[r].gram(mu, keys[r])
                if literal:
                    scores(0)
                keys[:, 0] = keys[:, 0].max()
                for t in range(1, m):
                    for r in range(P):
                        shards[r].pivot_column(t - 1, keys[r], cols[r])
                    pivot[: P * Bw].copy_(cols.reshape(-1))
                    for r in range(P):
                        if literal:
                            shards[r].colnorm(t, mu, pivot, keys[r], cn[r])
                        else:
                            shards[r].step(t, mu, pivot, keys[r])
                    if literal:
                        scores(t)
                    keys[:, t] = keys[:, t].max()

            rerun()
            # K4, as ShardedTed.select (both norm modes)
            for _ in range(m):
                cand = torch.zeros((P, m, 32), dtype=torch.int32, device=device)
                ncand = torch.zeros((P, m), dtype=torch.int32, device=device)
                for r in range(P):
                    shards[r].nearties(m, keys[r], cand[r], ncand[r])
                ca, na = cand.cpu().numpy().view(np.uint32), ncand.cpu().numpy()
                forced = [shards[r].refine(m, mu, keys[r], ca, na, P) for r in range(P)]
                assert all(np.array_equal(f, forced[0]) for f in forced), "shards disagree on K4"
                if len(forced[0]) == 0:
                    break
                rerun(forced[0])
            host = keys[0].cpu().numpy().view(np.uint64)
        for s in shards:
            s.check()
        if stats is not None:
            stats.update(L.bted_get_stats(shards[0].ctx))
        return L.decode_keys(host)
    finally:
        for s in shards:
            s.close()
