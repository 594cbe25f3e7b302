"""Seeded synthetic input generators shared by the oracle tests, the CUDA-path
tests and bench.py.

This module holds NO arithmetic of the method (no MLP forward/backward, no
softmax, no SGD, no batch-size rule).  It only produces datasets, labels and
initial parameters from fixed seeds, so that both sides of a parity test start
from identical inputs.  Recipes are documented in DESIGN.md section "Inputs".
"""
from .data import (  # noqa: F401
    DATASETS,
    bf16_round,
    covtype_like,
    delicious_like,
    init_params,
    make_dataset,
    pad_cols,
    params_to_flat,
    flat_to_params,
    sparse_like,
)
