"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This package holds NO arithmetic of the method (no Gram matrix, no score,
no deflation, no batch sampling): only the pools of encoded deployment
configurations the method is run on, and the RBF bandwidth chosen for them.
Both `oracle/` and the CUDA path consume what it produces.
"""
from .knob_pools import (  # noqa: F401
    ConvWorkload,
    KnobSpace,
    WORKLOADS,
    make_pool,
    uniform_pool,
    median_gamma,
    config_pool,
    CONFIGS,
    whole_model_nodes,
    whole_model_pools,
    MU,
)
