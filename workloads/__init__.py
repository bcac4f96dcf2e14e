"""Seeded synthetic inputs shared by the oracle, the tests and bench.py.

This package holds NO arithmetic of the triangular-solve method (no
substitution, no level sets, no reordering, no blocking).  It only draws
random sparse lower-triangular matrices with the shapes of the paper's
workloads ("lower triangular parts (plus a diagonal to avoid
singular)") and right-hand sides, so that the CUDA path and the oracle
consume byte-identical arrays.  The recipes are stated in DESIGN.md §4 and
SURVEY.md §8(d-2).
"""
from .generators import (  # noqa: F401
    CONFIGS,
    Matrix,
    gen_config,
    gen_rhs,
    gen_rhs_cols,
    gen_matrix,
    config_seed,
    c1_random,
    c2_laplacian_ic0,
    c3_powerlaw_layers,
    c4_supernodal,
    c5_random_multirhs,
    shape_diagonal,
    shape_bidiagonal,
    shape_dense_lower,
    shape_arrow,
    shape_paper_fig1,
    shape_random_small,
    to_upper,
)
