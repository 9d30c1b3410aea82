"""The one-process-per-GPU drivers (dist.py) with TWO real processes and the
real libbted kernels: both ranks on the one GPU of the test box, the exchanges
over a gloo process group (NCCL refuses two ranks on one device).  Checks the
multi-process control flow end to end -- the tile-sharded implicit engine (one q
all-reduce per step), the row bands (key max + pivot all-gather), batch
round-robin + merge (winner all-gather) -- against the single-process results,
bit for bit."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu
MU = float(np.float32(0.1))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class _HostStagedComm:
    """TorchComm's interface over gloo with the tensors staged through host
    memory (the device->host copy on the current stream orders it after the
    library's kernels, which run on that same stream)."""

    def __init__(self):
        import torch.distributed as dist
        self.dist, self.rank, self.world = dist, dist.get_rank(), dist.get_world_size()

    def _reduce(self, t, op):
        h = t.cpu()
        self.dist.all_reduce(h, op=op)
        t.copy_(h)

    def allreduce_max_(self, t):
        self._reduce(t, self.dist.ReduceOp.MAX)

    def allreduce_sum_(self, t):
        self._reduce(t, self.dist.ReduceOp.SUM)

    def allgather_(self, out, inp):
        h = out.cpu()
        self.dist.all_gather_into_tensor(h, inp.cpu())
        out.copy_(h)


def _worker(rank, world, port, out_dir):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch
    import torch.distributed as dist
    import paper_conf_date_sunbg021_b200 as bt
    from paper_conf_date_sunbg021_b200.dist import (LibIShard, LibShard, ShardedImplicitTed, ShardedTed, band,
                                                    run_batches_dp)
    from synth import KnobSpace, WORKLOADS, make_pool, median_gamma
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    comm = _HostStagedComm()
    st = torch.cuda.Stream(dev)
    _, X = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), 3001, 5)
    g = median_gamma(X, 5)
    res = {}
    # tile-sharded implicit engine
    sh = LibIShard(X, 3001, 16, g, rank, world, dev, st)
    try:
        idx, sc = ShardedImplicitTed(sh, 3001, comm, dev, st).select(40, MU)
    finally:
        sh.close()
    res["ishard_idx"], res["ishard_sc"] = idx, sc.view(np.uint32)
    # dense row bands (symmetric mode)
    r0, r1, _ = band(3001, world, rank)
    shd = LibShard(X, 3001, 16, g, r0, r1, dev, st)
    try:
        idx, sc = ShardedTed(shd, 3001, comm, dev, st).select(24, MU)
    finally:
        shd.close()
    res["band_idx"], res["band_sc"] = idx, sc.view(np.uint32)
    # batch round-robin + merge
    _, P = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), 20000, 6)
    gp = median_gamma(P, 6)
    with bt.CandidateSet(P, gp, num_batches=5, seed=3, device=0, stream=st.cuda_stream) as pool:
        with torch.cuda.stream(st):
            sel, _ = run_batches_dp(pool.ctx, 1024, 16, MU, 5, comm, dev)
    res["bted_sel"] = np.asarray(sel)
    np.savez(os.path.join(out_dir, f"rank{rank}.npz"), **res)
    dist.barrier()
    dist.destroy_process_group()


def test_two_processes_match_single_process(tmp_path, need_gpu):
    import torch.multiprocessing as mp
    import paper_conf_date_sunbg021_b200 as bt
    from paper_conf_date_sunbg021_b200 import _lib as L
    from paper_conf_date_sunbg021_b200.dist import isharded_select_loopback
    from synth import KnobSpace, WORKLOADS, make_pool, median_gamma
    import torch
    mp.spawn(_worker, args=(2, _port(), str(tmp_path)), nprocs=2, join=True)
    r = [np.load(tmp_path / f"rank{k}.npz") for k in range(2)]
    for key in r[0].files:                                    # every rank holds the same result
        assert np.array_equal(r[0][key], r[1][key]), key
    _, X = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), 3001, 5)
    g = median_gamma(X, 5)
    dev = torch.device("cuda", 0)
    idx, sc = isharded_select_loopback(X, g, 2, 40, MU, dev, torch.cuda.Stream(dev))
    assert np.array_equal(r[0]["ishard_idx"], idx) and np.array_equal(r[0]["ishard_sc"], sc.view(np.uint32))
    with bt.CandidateSet(X, g, flags=L.BTED_FLAG_DENSE | L.BTED_FLAG_NO_SMALL) as cs:
        idx, sc = cs.select(24, MU)
    assert np.array_equal(r[0]["band_idx"], idx) and np.array_equal(r[0]["band_sc"], sc.view(np.uint32))
    _, P = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), 20000, 6)
    with bt.CandidateSet(P, median_gamma(P, 6), num_batches=5, seed=3) as pool:
        sel, _ = pool.run_batches(1024, 16, MU)
    assert np.array_equal(r[0]["bted_sel"], sel)
