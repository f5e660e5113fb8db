"""Seeded synthetic inputs (graphs, features, labels, weights).

Shared by the oracle tests and the CUDA path; holds none of the method's
arithmetic (see rng.py)."""
