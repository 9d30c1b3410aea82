"""Host->device copy rates: torch pinned copy vs the library's bted_update
(from torch-pinned memory and from pageable numpy memory)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_date_sunbg021_b200 as bt
from paper_conf_date_sunbg021_b200 import _lib as L

P, d = 1 << 20, 16
X = np.random.default_rng(0).random((P, d)).astype(np.float32)
Xh = torch.from_numpy(X).pin_memory()
Xd = torch.empty_like(Xh, device="cuda")
st = torch.cuda.Stream()
for name, fn in [("torch pinned copy_", lambda: Xd.copy_(Xh, non_blocking=True))]:
    with torch.cuda.stream(st):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for _ in range(10):
            fn()
        e1.record(st)
        torch.cuda.synchronize()
    print(f"{name}: {X.nbytes * 10 / (e0.elapsed_time(e1) / 1e3) / 1e9:.1f} GB/s")
cs = bt.CandidateSet(X, 0.3, stream=st.cuda_stream)
pa = L.PinnedArray(X.shape)
pa.array[:] = X
for name, ptr in [("bted_update pinned(torch)", Xh.data_ptr()), ("bted_update pageable(numpy)", X.ctypes.data),
                  ("bted_update pinned(bted_host_alloc)", pa.ptr)]:
    for _ in range(3):
        L.bted_update(cs.ctx, ptr)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(10):
        L.bted_update(cs.ctx, ptr)
    e1.record(st)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    L.bted_update(cs.ctx, ptr)
    torch.cuda.synchronize()
    print(f"{name}: {X.nbytes * 10 / (e0.elapsed_time(e1) / 1e3) / 1e9:.1f} GB/s (events); "
          f"single call wall {1e3 * (time.perf_counter() - t0):.2f} ms")
