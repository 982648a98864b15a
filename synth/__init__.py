"""Seeded synthetic inputs shaped like the paper's workloads (Table 2).

This package is INPUT GENERATION ONLY: it holds none of the SpMV method's arithmetic
(no blocking, no flags, no products).  Both the oracle side (tests/) and the product
side (bench.py) draw their inputs from here; nothing here imports either of them.
The recipes are stated in DESIGN.md ("Input recipe").
"""
from .matrices import (CSR, CONFIGS, laplacian_2d, dense, fem_like, webbase_like,
                       circuit_like, circuit_like_rows, random_tiny, random_coo, make_x,
                       config_matrix)

__all__ = ["CSR", "CONFIGS", "laplacian_2d", "dense", "fem_like", "webbase_like",
           "circuit_like", "circuit_like_rows", "random_tiny", "random_coo", "make_x",
           "config_matrix"]
