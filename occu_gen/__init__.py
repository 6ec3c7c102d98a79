"""Seeded synthetic input generators (graphs, Table I features, weights).

Shared by the tests, the oracle's callers and bench.py.  By design this package
holds none of the GNN's arithmetic.
"""
from . import configs, dags, features, prng, weights  # noqa: F401
