"""Seeded synthetic input generators shared by the oracle tests, the CUDA parity
tests and bench.py.

This package holds ONLY input construction (weight matrices of the paper's
three workload families and random bit vectors).  It contains none of the
method's arithmetic (no energies, no deltas, no search, no GA), so it can be
used by both sides of the parity check without coupling them.
"""
from .generators import (  # noqa: F401
    random_qubo,
    random_qubo_ctr,
    random_qubo_ctr_rows,
    maxcut_graph,
    maxcut_qubo,
    tsp_instance,
    tsp_qubo,
    random_solutions,
    words_per_vector,
    pack_bits,
    unpack_bits,
)
