"""The multi-GPU drivers over a REAL NCCL process group (one rank: this run has
one GPU).  Exercises dist.TorchComm's NCCL all-reduce / all-gather on CUDA
tensors, stream ordering between them and libbted's kernels, and checks the
results against the single-GPU entry points bit for bit."""
import os
import socket

import numpy as np
import pytest

import paper_conf_date_sunbg021_b200 as bt
from paper_conf_date_sunbg021_b200 import _lib as L
from synth import KnobSpace, WORKLOADS, make_pool, median_gamma

pytestmark = pytest.mark.gpu
MU = float(np.float32(0.1))


@pytest.fixture(scope="module")
def nccl_group(need_gpu):
    import torch
    import torch.distributed as dist
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
    yield dev
    dist.destroy_process_group()


@pytest.mark.parametrize("graph", [False, True], ids=["eager", "cuda-graph"])
def test_sharded_ted_over_nccl_matches_dense_select(nccl_group, graph):
    import torch
    from paper_conf_date_sunbg021_b200.dist import LibShard, ShardedTed, TorchComm, band
    _, X = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), 5000, 3)
    g = median_gamma(X, 3)
    with bt.CandidateSet(X, g, flags=L.BTED_FLAG_DENSE | L.BTED_FLAG_NO_SMALL) as cs:
        idx, sc = cs.select(32, MU)
    comm = TorchComm()
    st_ = torch.cuda.Stream(nccl_group)
    r0, r1, _ = band(5000, comm.world, comm.rank)
    shard = LibShard(X, 5000, 16, g, r0, r1, nccl_group, st_)
    try:
        sted = ShardedTed(shard, 5000, comm, nccl_group, st_, graph=graph)
        sidx, ssc = sted.select(32, MU)
        sidx2, _ = sted.select(32, MU)                        # replay (graph) / rerun (eager)
        assert np.array_equal(sidx2, sidx)
    finally:
        shard.close()
    assert np.array_equal(sidx, idx)
    assert np.array_equal(ssc.view(np.uint32), sc.view(np.uint32))


@pytest.mark.parametrize("graph", [False, True], ids=["eager", "cuda-graph"])
def test_sharded_ted_literal_norms_over_nccl(nccl_group, graph):
    """norm_mode='literal': the partial column norms go through a real NCCL all-reduce(SUM)."""
    import torch
    from oracle import literal
    from tests.parity import GAP_K4, check_ted
    from paper_conf_date_sunbg021_b200.dist import LibShard, ShardedTed, TorchComm, band
    N = 3000
    _, X = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), N, 4)
    g = median_gamma(X, 4)
    comm = TorchComm()
    st_ = torch.cuda.Stream(nccl_group)
    r0, r1, _ = band(N, comm.world, comm.rank)
    shard = LibShard(X, N, 16, g, r0, r1, nccl_group, st_)
    try:
        sted = ShardedTed(shard, N, comm, nccl_group, st_, graph=graph, norm_mode="literal")
        sidx, ssc = sted.select(24, MU)
        sidx2, ssc2 = sted.select(24, MU)
        assert np.array_equal(sidx2, sidx) and np.array_equal(ssc2, ssc)
    finally:
        shard.close()
    tr = literal.ted(X, g, MU, 24, forced=sidx.tolist())
    check_ted(sidx, ssc, tr, "nccl-literal", gap_exact=GAP_K4)   # K4 in the literal mode too


@pytest.mark.parametrize("graph", [False, True], ids=["eager", "cuda-graph"])
def test_tile_sharded_implicit_over_nccl(nccl_group, graph):
    """ShardedImplicitTed: the per-step q all-reduce goes through real NCCL (one rank)."""
    import torch
    from oracle import dense
    from tests.parity import GAP_K4, check_ted
    from paper_conf_date_sunbg021_b200.dist import LibIShard, ShardedImplicitTed, TorchComm
    N = 5000
    _, X = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), N, 5)
    g = median_gamma(X, 5)
    comm = TorchComm()
    st_ = torch.cuda.Stream(nccl_group)
    be = LibIShard(X, N, 16, g, comm.rank, comm.world, nccl_group, st_)
    try:
        sted = ShardedImplicitTed(be, N, comm, nccl_group, st_, graph=graph)
        idx, sc = sted.select(32, MU)
        idx2, sc2 = sted.select(32, MU)
        assert np.array_equal(idx2, idx) and np.array_equal(sc2, sc)
    finally:
        be.close()
    check_ted(idx, sc, dense.ted(X, g, MU, 32, forced=idx), "nccl-ishard", gap_exact=GAP_K4)


def test_batch_round_robin_over_nccl_matches_run_batches(nccl_group):
    import torch
    from paper_conf_date_sunbg021_b200.dist import TorchComm, run_batches_dp
    _, X = make_pool(KnobSpace(WORKLOADS["vgg16_conv1_1"], 16), 40000, 9)
    g = median_gamma(X, 9)
    st_ = torch.cuda.Stream(nccl_group)
    with bt.CandidateSet(X, g, num_batches=3, seed=5, stream=st_.cuda_stream) as pool:
        ref, _ = pool.run_batches(2000, 16, MU)
        with torch.cuda.stream(st_):
            sel, win = run_batches_dp(pool.ctx, 2000, 16, MU, 3, TorchComm(), nccl_group)
    assert np.array_equal(sel, ref)
