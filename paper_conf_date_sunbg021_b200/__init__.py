"""B200-native BTED (batch transductive experimental design) hot path.

Sun, Bai, Geng, Yu, "Deep Neural Network Hardware Deployment Optimization via
Advanced Active Learning", DATE 2021 -- Algorithms 1 and 2.

The compute lives in libbted.so (hand-written sm_100a CUDA behind the C ABI
of include/bted.h); this package is its thin binding (`_lib`, same names as
the C ABI), a small object wrapper (`api`) and the multi-GPU drivers built on
torch.distributed (`dist`).  There is no CPU fallback.
"""
from . import _lib  # noqa: F401
from ._lib import (  # noqa: F401
    BTED_KERNEL_RBF, BTED_KERNEL_LINEAR, BTED_FLAG_NO_GRAPH, BTED_FLAG_NO_SMALL, BTED_FLAG_LITERAL,
    BTED_FLAG_DENSE, BTED_FLAG_NO_REFINE, BTED_FLAG_LOOPBACK, BTED_FLAG_NCCL, BtedError, default_params,
    bted_create, bted_select, bted_run_batches, bted_batch_teds, bted_merge,
    bted_sample_batches, bted_shard_create, bted_shard_gram, bted_shard_step,
    bted_shard_pivot_column, bted_shard_ld, bted_shard_check, bted_destroy,
    bted_kernel_launches, decode_keys,
)
from .api import CandidateSet  # noqa: F401

__all__ = [
    "CandidateSet", "BtedError", "default_params", "bted_create", "bted_select",
    "bted_run_batches", "bted_batch_teds", "bted_merge", "bted_sample_batches",
    "bted_shard_create", "bted_shard_gram", "bted_shard_step", "bted_shard_pivot_column",
    "bted_shard_ld", "bted_shard_check", "bted_destroy", "bted_kernel_launches",
]
