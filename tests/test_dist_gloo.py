"""World-size-2 CPU (gloo) tests of the multi-GPU exchange protocols in
paper_conf_date_sunbg021_b200/dist.py.  The per-rank compute is replaced by
test-only numpy backends (fp64, this file); the drivers, band bookkeeping,
padding and collectives are the product code.  The GPU kernels behind the
same protocol are covered by test_gpu_parity.py::test_row_sharded_loopback_*.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import literal
from oracle.sampling import sample_batches
from synth import KnobSpace, WORKLOADS, make_pool, median_gamma
from tests.parity import check_ted

MU = float(np.float32(0.1))


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def pack(score: float, idx: int) -> int:
    bits = int(np.float32(score).view(np.uint32))
    return ((bits + 1) << 32) | (0xFFFFFFFF - idx)


def unpack_idx(key: int) -> int:
    return 0xFFFFFFFF - (int(key) & 0xFFFFFFFF)


class NumpyShard:
    """Test-only band backend: rows [row0, row1) of Alg. 1 in fp64."""

    def __init__(self, X, gamma, row0, row1):
        self.X = X.astype(np.float64)
        self.g, self.r0, self.r1 = gamma, row0, row1
        self.N = X.shape[0]
        self.ld = self.N
        self.sel = np.zeros(row1 - row0, bool)

    def _key(self, t, keys, s_prev=None):
        g = (self.K * self.K).sum(1)
        diag = self.K[np.arange(self.r1 - self.r0), np.arange(self.r0, self.r1)]
        score = g / (diag + self.mu)
        best = 0
        for lr in range(self.r1 - self.r0):
            if not self.sel[lr]:
                best = max(best, pack(score[lr], self.r0 + lr))
        keys[t] = max(int(keys[t]), best)

    def gram(self, mu, keys):
        self.mu = mu
        d2 = ((self.X[self.r0:self.r1, None, :] - self.X[None, :, :]) ** 2).sum(-1)
        self.K = np.exp(-self.g * d2)
        self.sel[:] = False
        self._key(0, keys)

    def pivot_column(self, t, keys, col):
        s = unpack_idx(int(keys[t]))
        col.zero_()
        col[: self.r1 - self.r0] = torch.from_numpy(self.K[:, s].astype(np.float32))
        self.Kcol64 = self.K[:, s].copy()

    def step(self, t, mu, pivot, keys):
        s = unpack_idx(int(keys[t - 1]))
        p = pivot[: self.N].numpy().astype(np.float64)
        # the gathered pivot row is fp32 on the wire (as on the GPU path)
        a = p[self.r0:self.r1].copy()
        if self.r0 <= s < self.r1:
            self.sel[s - self.r0] = True                  # l.4: X = X u x
        self.K -= np.outer(a, p) / (p[s] + mu)           # l.5 on the band
        self._key(t, keys)                                # next l.3 over unselected rows

    def colnorm(self, t, mu, pivot, keys, cn):
        """Literal norm mode: (t > 0) l.5 on the band, then the band's part of every column norm."""
        if t > 0:
            s = unpack_idx(int(keys[t - 1]))
            p = pivot[: self.N].numpy().astype(np.float64)
            if self.r0 <= s < self.r1:
                self.sel[s - self.r0] = True
            self.K -= np.outer(p[self.r0:self.r1], p) / (p[s] + mu)
        cn.zero_()
        cn[: self.N] = torch.from_numpy((self.K * self.K).sum(0))

    def scores(self, t, mu, cn, keys):
        g = cn[self.r0:self.r1].numpy().astype(np.float64)           # all-reduced column norms
        diag = self.K[np.arange(self.r1 - self.r0), np.arange(self.r0, self.r1)]
        score = g / (diag + mu)
        best = 0
        for lr in range(self.r1 - self.r0):
            if not self.sel[lr]:
                best = max(best, pack(score[lr], self.r0 + lr))
        keys[t] = max(int(keys[t]), best)

    def check(self):
        pass


def _shard_worker(rank, world, port, X, gamma, m, q, norm_mode="symmetric"):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_date_sunbg021_b200.dist import ShardedTed, TorchComm, band
    comm = TorchComm()
    r0, r1, _ = band(X.shape[0], world, rank)
    st = ShardedTed(NumpyShard(X, gamma, r0, r1), X.shape[0], comm, torch.device("cpu"), norm_mode=norm_mode)
    idx, score = st.select(m, MU)
    q.put((rank, idx.tolist(), score.tolist()))
    dist.destroy_process_group()


def _run(world, target, *args, **kw):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=target, args=(r, world, port, *args, q), kwargs=kw) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=300) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return sorted(out)


def test_sharded_protocol_two_ranks_matches_oracle_and_one_rank():
    _, X = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), 301, 12)   # ragged: 301 rows / 2
    g = median_gamma(X, 12)
    m = 12
    two = _run(2, _shard_worker, X, g, m)
    one = _run(1, _shard_worker, X, g, m)
    assert two[0][1] == two[1][1] == one[0][1]               # every rank decodes the same selection
    tr = literal.ted(X, g, MU, m, forced=two[0][1])
    check_ted(np.array(two[0][1]), np.array(two[0][2]), tr, "gloo-shard")


def test_sharded_literal_column_norm_exchange_two_ranks():
    """norm_mode='literal': all-reduce(SUM) of partial column norms (north_star), same picks."""
    _, X = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), 301, 12)
    g = median_gamma(X, 12)
    m = 12
    lit = _run(2, _shard_worker, X, g, m, norm_mode="literal")
    sym = _run(2, _shard_worker, X, g, m)
    assert lit[0][1] == lit[1][1] == sym[0][1]
    tr = literal.ted(X, g, MU, m, forced=lit[0][1])
    check_ted(np.array(lit[0][1]), np.array(lit[0][2]), tr, "gloo-shard-literal")


class NumpyIShard:
    """Test-only tile-shard backend of ShardedImplicitTed, fp64 numpy: this rank
    owns the entries (i, j) of the 128 x 128 tiles (min(I,J), max(I,J)) whose
    row-major upper-triangle index is rank (mod P); everything else (the factor
    L, running norms n_v and diagonal r_vv) is replicated, as in libbted."""

    T = 128

    def __init__(self, X, gamma, rank, nranks):
        X = X.astype(np.float64)
        self.N = X.shape[0]
        d2 = ((X[:, None, :] - X[None, :, :]) ** 2).sum(-1)
        K = np.exp(-gamma * d2)
        nT = -(-self.N // self.T)
        blk = np.arange(self.N) // self.T
        lo, hi = np.minimum.outer(blk, blk), np.maximum.outer(blk, blk)
        toff = lo * nT - lo * (lo - 1) // 2 + (hi - lo)           # tile index of entry (i, j)
        self.Kown = np.where(toff % nranks == rank, K, 0.0)      # this rank's share of K
        self.diag = np.diag(K).copy()
        self.qlen = self.N

    def _put_key(self, t, keys):
        score = np.maximum(self.n, 0.0) / (self.r + self.mu)              # as libbted's fin64
        best = 0
        for i in range(self.N):
            if not self.sel[i]:
                best = max(best, pack(score[i], i))
        keys[t] = best

    def head(self, m, mu, q):
        self.mu, self.L = mu, []
        self.sel = np.zeros(self.N, bool)
        q.zero_()
        q[: self.N] = torch.from_numpy((self.Kown * self.Kown).sum(1))       # own part of ||K_:v||^2

    def fin(self, t, mu, q, keys):
        qv = q[: self.N].numpy().astype(np.float64)
        if t == 0:
            self.n, self.r = qv.copy(), self.diag.copy()
        else:
            l = self.L[-1]
            Lp = np.array(self.L[:-1]).T if len(self.L) > 1 else np.zeros((self.N, 0))
            Rl = qv - Lp @ (Lp.T @ l)                              # (R l)_v = (K l)_v - L (L^T l)
            self.n = self.n - 2 * l * Rl + l * l * (l @ l)
            self.r = self.r - l * l
        self._put_key(t, keys)

    def step(self, t, mu, keys, q):
        s = unpack_idx(int(keys[t - 1]))
        self.sel[s] = True
        Kcol = self.Kfull_col(s)
        Lm = np.array(self.L).T if self.L else np.zeros((self.N, 0))
        l = (Kcol - Lm @ Lm[s]) / np.sqrt(self.r[s] + mu)
        self.L.append(l)
        q.zero_()
        q[: self.N] = torch.from_numpy(self.Kown @ l)                      # own part of K l (mask symmetric)

    def Kfull_col(self, s):
        return self._K[:, s]

    def check(self):
        pass


def _ishard_worker(rank, world, port, X, gamma, m, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_date_sunbg021_b200.dist import ShardedImplicitTed, TorchComm
    be = NumpyIShard(X, gamma, rank, world)
    Xd = X.astype(np.float64)
    be._K = np.exp(-gamma * ((Xd[:, None, :] - Xd[None, :, :]) ** 2).sum(-1))   # column s (replicated X)
    st = ShardedImplicitTed(be, X.shape[0], TorchComm(), torch.device("cpu"))
    idx, score = st.select(m, MU)
    q.put((rank, idx.tolist(), score.tolist()))
    dist.destroy_process_group()


def test_tile_sharded_implicit_protocol_two_ranks():
    """ShardedImplicitTed: one all-reduce(SUM) of the partial q per step; every
    rank decodes the same picks, equal to one rank's and to the oracle's."""
    _, X = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), 300, 14)   # 3 blocks of 128: 6 tiles
    g = median_gamma(X, 14)
    m = 12
    two = _run(2, _ishard_worker, X, g, m)
    one = _run(1, _ishard_worker, X, g, m)
    assert two[0][1] == two[1][1] == one[0][1]
    tr = literal.ted(X, g, MU, m, forced=two[0][1])
    check_ted(np.array(two[0][1]), np.array(two[0][2]), tr, "gloo-ishard")


class NumpyPool:
    """Test-only batch backend: Alg. 2 l.1-4 / l.5-6 by the oracle."""

    def __init__(self, X, gamma, B, seed):
        self.X, self.g, self.B, self.seed = X, gamma, B, seed

    def batch_teds(self, M, m, mu, b_begin, b_step, out):
        batches = sample_batches(self.X.shape[0], M, self.B, self.seed)
        k = 0
        for b in range(b_begin, self.B, b_step):
            tr = literal.ted(self.X[batches[b]], self.g, mu, m)
            out[k * m:(k + 1) * m] = torch.from_numpy(batches[b][np.array(tr.idx)])
            k += 1

    def merge(self, winners, m, mu):
        w = winners.numpy()
        XU = np.unique(w[w >= 0])
        tr = literal.ted(self.X[XU], self.g, mu, min(m, len(XU)))
        return XU[np.array(tr.idx)]


def _dp_worker(rank, world, port, X, gamma, B, M, m, seed, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_date_sunbg021_b200.dist import TorchComm, run_batches_dp
    sel, win = run_batches_dp(NumpyPool(X, gamma, B, seed), M, m, MU, B, TorchComm(), torch.device("cpu"))
    q.put((rank, [int(x) for x in sel], win.tolist()))
    dist.destroy_process_group()


@pytest.mark.parametrize("B", [3, 4])
def test_batch_round_robin_two_ranks_equals_single_process_bted(B):
    _, X = make_pool(KnobSpace(WORKLOADS["vgg16_conv1_1"], 16), 3000, 5)
    g = median_gamma(X, 5)
    M, m, seed = 200, 8, 21
    out = _run(2, _dp_worker, X, g, B, M, m, seed)
    batches = sample_batches(X.shape[0], M, B, seed)
    ref_sel, ref_win, _, _, _ = literal.bted(X, batches, g, MU, m)
    assert out[0][1] == out[1][1] == ref_sel.tolist()
    # batch b ran on rank b mod 2, in slot b // 2; a rank with fewer batches pads with -1
    for b in range(B):
        r, k = b % 2, b // 2
        assert out[r][2][k * m:(k + 1) * m] == ref_win[b].tolist()
    if B % 2:
        assert out[1][2][-m:] == [-1] * m
