"""Seeded synthetic input generators shared by the oracle tests, the GPU parity
tests and bench.py.

This module builds INPUTS only: CSR matrices (row offsets, column indices,
values) and dense vectors with the shapes and structure of the BASELINE.json
workloads (C1-C5).  It contains none of the method's arithmetic (no SpMV,
SpAdd or SpGEMM), so that neither side of a parity check can borrow from the
other through it.  Recipes are restated in DESIGN.md §3.
"""
from .matrices import (  # noqa: F401
    CSR,
    poisson2d_5pt,
    poisson3d_27pt,
    rmat,
    pathological,
    random_rows,
    random_csr,
    transpose,
    identity,
    x_vector,
    int_values,
    config,
    CONFIGS,
)
