"""Seeded synthetic inputs (graphs, orders, placements) shared by the oracle tests and the
CUDA tests.  No arithmetic of the method lives here (see rng.py / dag.py / shaped.py)."""
