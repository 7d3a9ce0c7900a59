"""Seeded synthetic inputs shared by the oracle tests, the GPU tests and bench.py.

This module holds NONE of the method's arithmetic (no sampling, dedup, time
encoding or attention).  It only draws graphs, features, weights and batches
with the shapes of the paper's workloads (Table 3; batch
sizes P:407) and the value distributions stated in DESIGN.md §3.
"""
from .configs import CONFIGS, Config, get_config  # noqa: F401
from .gen import (  # noqa: F401
    Graph,
    make_graph,
    make_negatives,
    make_layer_params,
    model_params,
    feature_table,
    make_time_params,
    batch_roots_inputs,
    feature_rows,
    make_gru_params,
)
