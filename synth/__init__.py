"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and
bench.py.  Holds no arithmetic of the method (no rounding, no DP) — only the
pinned generator of SURVEY.md §8(d) and the workload table."""
from .instances import WORKLOADS, Workload, jobs, dstar  # noqa: F401
