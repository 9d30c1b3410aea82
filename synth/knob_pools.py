"""Synthetic pools of encoded AutoTVM conv2d deployment configurations.

What the paper fixes (PAPER.md, /root/reference):
  * Def. 1 (Sec. II-D): a deployment configuration is "encoded
    as the attributes of a feature vector" -- the encoding itself is not given.
  * The config space of one node is huge: "the first optimization node in
    VGG-16 has approximately 0.2 billion configuration points"
    and ">50 million" on average.
  * The knobs are CUDA schedule knobs: thread binding, thread cooperation,
    memory locality, tensorization (Fig. 2).

Reading adopted: the AutoTVM
``conv2d_direct`` CUDA template knob structure, which reproduces the paper's
VGG-16 figure exactly (202,309,632 points for conv1_1, checked in
tests/test_synth.py):
  tile_f, tile_y, tile_x  = ordered 4-way factorisations of C_out, H_out, W_out
  tile_rc, tile_ry, tile_rx = ordered 2-way factorisations of C_in, KH, KW
  auto_unroll_max_step in {0, 512, 1500}; unroll_explicit in {0, 1}.
Encoding: log2(factor)/log2(dim) of the first 3 factors of each 4-way split and
of the first factor of each 2-way split (d = 12; a split of dim 1 encodes 0),
plus a one-hot of auto_unroll_max_step (3) and unroll_explicit (1) -> d = 16.

This module contains no arithmetic of the BTED method itself.
"""
from __future__ import annotations

import math
from dataclasses import dataclass
from functools import lru_cache

import numpy as np

__all__ = [
    "ConvWorkload", "KnobSpace", "WORKLOADS", "make_pool", "uniform_pool",
    "median_gamma", "config_pool", "CONFIGS", "ordered_factorizations",
    "whole_model_nodes", "whole_model_pools", "MU",
]


@dataclass(frozen=True)
class ConvWorkload:
    name: str
    c_out: int
    h_out: int
    w_out: int
    c_in: int
    kh: int
    kw: int
    depthwise: bool = False


@lru_cache(maxsize=None)
def ordered_factorizations(n: int, k: int) -> tuple:
    """All ordered k-tuples of positive integers whose product is n."""
    if k == 1:
        return ((n,),)
    out = []
    for f in range(1, n + 1):
        if n % f == 0:
            for rest in ordered_factorizations(n // f, k - 1):
                out.append((f,) + rest)
    return tuple(out)


def _split_features(dim: int, parts: int) -> np.ndarray:
    """Feature rows of every ordered `parts`-way split of `dim` (fp64)."""
    facts = ordered_factorizations(dim, parts)
    nf = parts - 1 if parts > 2 else 1
    rows = np.zeros((len(facts), nf), dtype=np.float64)
    if dim > 1:
        ld = math.log2(dim)
        for r, f in enumerate(facts):
            for c in range(nf):
                rows[r, c] = math.log2(f[c]) / ld
    return rows


UNROLL_STEPS = (0, 512, 1500)
UNROLL_EXPLICIT = (0, 1)


class KnobSpace:
    """Mixed-radix enumeration of one conv2d node's knob space.

    A config index in [0, size) decodes digit by digit (last knob fastest)
    into one knob choice per knob; ``features`` maps indices to fp32 rows.
    """

    def __init__(self, wl: ConvWorkload, d: int = 16):
        if d not in (12, 16):
            raise ValueError("d must be 12 or 16")
        self.wl = wl
        self.d = d
        tables = [
            _split_features(wl.c_out, 4),
            _split_features(wl.h_out, 4),
            _split_features(wl.w_out, 4),
        ]
        if wl.depthwise:
            # depthwise nodes have no reduction splits; their features are 0
            tables += [np.zeros((1, 1)), np.zeros((1, 1)), np.zeros((1, 1))]
        else:
            tables += [
                _split_features(wl.c_in, 2),
                _split_features(wl.kh, 2),
                _split_features(wl.kw, 2),
            ]
        unroll = np.eye(3, dtype=np.float64)
        expl = np.array([[0.0], [1.0]])
        if d == 12:
            # the unroll knobs stay in the space but not in the encoding
            unroll = np.zeros((3, 0))
            expl = np.zeros((2, 0))
        tables += [unroll, expl]
        self.tables = tables
        self.radices = [t.shape[0] for t in tables]
        self.size = int(np.prod([int(r) for r in self.radices], dtype=object))

    def digits(self, idx: np.ndarray) -> list:
        idx = np.asarray(idx, dtype=np.int64).copy()
        out = [None] * len(self.radices)
        for k in range(len(self.radices) - 1, -1, -1):
            out[k] = idx % self.radices[k]
            idx //= self.radices[k]
        return out

    def features(self, idx: np.ndarray) -> np.ndarray:
        dig = self.digits(idx)
        cols = [t[dg] for t, dg in zip(self.tables, dig)]
        X = np.concatenate(cols, axis=1)
        assert X.shape[1] == self.d
        return np.ascontiguousarray(X.astype(np.float32))


# Conv workloads (C_out, H_out, W_out, C_in, KH, KW) at 224x224, batch 1.
WORKLOADS = {
    "vgg16_conv1_1": ConvWorkload("vgg16_conv1_1", 64, 224, 224, 3, 3, 3),
    "resnet18_layer1": ConvWorkload("resnet18_layer1", 64, 56, 56, 64, 3, 3),
}


def _resnet50_nodes():
    """Unique conv2d workloads of ResNet-50 (torchvision layout), forward order."""
    wl = [(64, 112, 112, 3, 7, 7)]
    cfg = [(64, 56, 3), (128, 28, 4), (256, 14, 6), (512, 7, 3)]
    cin = 64
    for width, hw, _blocks in cfg:
        out = width * 4
        first_hw = hw * 2 if width != 64 else hw
        # first block: 1x1 reduce (at the input resolution), 3x3 (stride on v1.5), 1x1 expand, downsample
        wl += [(width, first_hw, first_hw, cin, 1, 1), (width, hw, hw, width, 3, 3),
               (out, hw, hw, width, 1, 1), (out, hw, hw, cin, 1, 1)]
        # remaining blocks: 1x1 reduce from `out`, 3x3, 1x1 expand
        wl += [(width, hw, hw, out, 1, 1)]
        cin = out
    seen, uniq = set(), []
    for w in wl:
        if w not in seen:
            seen.add(w)
            uniq.append(w)
    return [ConvWorkload(f"resnet50_n{i}", *w) for i, w in enumerate(uniq)]


def _mobilenet_v2_nodes():
    """Unique conv2d workloads of MobileNet-v2 (1.0, 224), forward order."""
    wl = [((32, 112, 112, 3, 3, 3), False)]
    # (expansion t, out c, repeats n, stride s)
    cfg = [(1, 16, 1, 1), (6, 24, 2, 2), (6, 32, 3, 2), (6, 64, 4, 2),
           (6, 96, 3, 1), (6, 160, 3, 2), (6, 320, 1, 1)]
    cin, hw = 32, 112
    for t, c, n, s in cfg:
        for i in range(n):
            stride = s if i == 0 else 1
            hid = cin * t
            if t != 1:
                wl.append(((hid, hw, hw, cin, 1, 1), False))
            ohw = hw // stride
            wl.append(((hid, ohw, ohw, 1, 3, 3), True))   # depthwise 3x3
            wl.append(((c, ohw, ohw, hid, 1, 1), False))
            cin, hw = c, ohw
    wl.append(((1280, 7, 7, 320, 1, 1), False))
    seen, uniq = set(), []
    for w in wl:
        if w not in seen:
            seen.add(w)
            uniq.append(w)
    return [ConvWorkload(f"mobilenetv2_n{i}", *w, depthwise=dw)
            for i, (w, dw) in enumerate(uniq)]


def whole_model_nodes(per_model: int = 20):
    """'~40 tunable nodes': the first `per_model` unique workloads of each model."""
    return _resnet50_nodes()[:per_model] + _mobilenet_v2_nodes()[:per_model]


def make_pool(space: KnobSpace, P: int, seed: int) -> tuple:
    """P distinct config indices drawn uniformly from the space (sorted), and
    their fp32 features.  P is clipped to the space size."""
    P = min(int(P), space.size)
    rng = np.random.default_rng(seed)
    if P == space.size:
        idx = np.arange(P, dtype=np.int64)
    else:
        idx = np.sort(rng.choice(space.size, size=P, replace=False).astype(np.int64))
    return idx, space.features(idx)


def uniform_pool(P: int, d: int, seed: int) -> np.ndarray:
    """Control pool: iid uniform [0, 1)^d rows, fp32."""
    rng = np.random.default_rng(seed)
    return rng.random((P, d)).astype(np.float32)


def median_gamma(X: np.ndarray, seed: int, n_sub: int = 2000) -> float:
    """RBF bandwidth gamma = 1 / median ||x_i - x_j||^2 over a seeded subsample
    (reading A2 in DESIGN.md: the paper gives no bandwidth).  Returned as the
    fp32 value both sides use."""
    rng = np.random.default_rng(seed + 0x9E37)
    n = X.shape[0]
    sub = X[rng.choice(n, size=min(n_sub, n), replace=False)].astype(np.float64)
    sq = (sub * sub).sum(1)
    d2 = sq[:, None] + sq[None, :] - 2.0 * sub @ sub.T
    iu = np.triu_indices(sub.shape[0], 1)
    med = float(np.median(np.maximum(d2[iu], 0.0)))
    if not med > 0.0:
        med = 1.0
    return float(np.float32(1.0 / med))


# The BASELINE.json configurations; mu = 0.1.
CONFIGS = {
    "toy": dict(workload="resnet18_layer1", d=12, pool=256, M=256, B=1, m=16, seed=0),
    "resnet18": dict(workload="resnet18_layer1", d=16, pool=1 << 20, M=16384, B=1, m=64, seed=18),
    "vgg16": dict(workload="vgg16_conv1_1", d=16, pool=1 << 20, M=32768, B=8, m=64, seed=16),
    "oversized": dict(workload="vgg16_conv1_1", d=16, pool=1 << 20, M=65536, B=1, m=64, seed=65536),
    "paper": dict(workload="vgg16_conv1_1", d=16, pool=1 << 20, M=500, B=10, m=64, seed=2021),
    # one un-batched TED on 131072 points (K = 34 GB packed per buffer)
    "large": dict(workload="vgg16_conv1_1", d=16, pool=1 << 20, M=131072, B=1, m=64, seed=131072),
    # ResNet-50 + MobileNet-v2: 40 nodes x 4 batches of 32768 (whole_model_pools)
    "wholemodel": dict(workload="resnet50+mobilenetv2 (40 nodes)", d=16, pool=1 << 20, M=32768, B=4, m=64, seed=5000),
}
MU = 0.1


def whole_model_pools(pool: int = 1 << 20, d: int = 16, which=None):
    """[(node, X fp32 [P_node, d], gamma)] for the 'wholemodel' config: the first
    20 unique conv workloads of ResNet-50 and of MobileNet-v2, pool P =
    min(pool, |D|) each, seed = 5000 + node index.
    which: the node indices (into whole_model_nodes()) to build; default all."""
    nodes = whole_model_nodes()
    out = []
    for k in (range(len(nodes)) if which is None else which):
        space = KnobSpace(nodes[k], d)
        _, X = make_pool(space, pool, 5000 + k)
        out.append((nodes[k], X, median_gamma(X, 5000 + k)))
    return out


def config_pool(name: str, pool: int | None = None):
    """(X pool fp32 [P, d], gamma fp32, cfg dict) for a named configuration."""
    cfg = dict(CONFIGS[name])
    cfg["mu"] = MU
    if pool is not None:
        cfg["pool"] = int(pool)
    space = KnobSpace(WORKLOADS[cfg["workload"]], cfg["d"])
    _, X = make_pool(space, cfg["pool"], cfg["seed"])
    cfg["pool"] = X.shape[0]
    gamma = median_gamma(X, cfg["seed"])
    return X, gamma, cfg
