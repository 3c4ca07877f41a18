"""Pinned instance generator and workload table.

Processing times are uniform random integers, as in the paper's experiments
("The problem instances are generated using the uniform distribution and
considering different numbers of jobs and machines"), drawn as
``numpy.random.default_rng(seed).integers(1, P, size=n, endpoint=True)``.

The literal BASELINE.json configs 2-5 have n/m >= 20, so no job is long at any
T in [LB, UB] and the DP is empty; the "shaped" twins keep
n, eps and U{1..1000} and re-choose m so the k-dimensional DP is non-trivial.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


def jobs(n: int, P: int, seed: int) -> np.ndarray:
    """p_j ~ U{1..P}, int64, pinned RNG."""
    return np.random.default_rng(seed).integers(1, P, size=n, endpoint=True).astype(np.int64)


@dataclass(frozen=True)
class Workload:
    name: str
    n: int
    m: int
    eps: float
    P: int
    seed: int
    role: str

    def p(self) -> np.ndarray:
        return jobs(self.n, self.P, self.seed)


WORKLOADS = {w.name: w for w in [
    Workload("M1", 12, 3, 0.3, 100, 0, "cfg1 literal: brute-force parity (seeds 0-999)"),
    Workload("M2", 200, 10, 0.3, 100, 0, "cfg2 literal: empty-DP path"),
    Workload("M2s", 200, 60, 0.3, 1000, 2, "cfg2 shaped: 1-GPU level-fill baseline"),
    Workload("M3", 1000, 20, 0.2, 1000, 0, "cfg3 literal: empty-DP path"),
    Workload("M3s", 1000, 172, 0.2, 1000, 0, "cfg3 shaped"),
    Workload("M3g", 1000, 184, 0.2, 1000, 1, "cfg3 'table ~GB'"),
    Workload("M4", 5000, 50, 0.15, 1000, 0, "cfg4 literal: empty-DP path"),
    Workload("M4s", 200, 30, 0.15, 1000, 0, "cfg4 shaped, K=7"),
    Workload("M4x", 200, 31, 0.15, 1000, 0, "largest-dimension instance (K=8)"),
    Workload("M5", 2000, 30, 0.3, 1000, 0, "cfg5 literal: empty-DP path"),
    Workload("M5s-0.3", 2000, 435, 0.3, 1000, 0, "cfg5 shaped multi-section sweep"),
    Workload("M5s-0.2", 2000, 320, 0.2, 1000, 0, "cfg5 shaped multi-section sweep"),
    Workload("M5s-0.15", 2000, 210, 0.15, 1000, 0, "cfg5 shaped multi-section sweep"),
]}


def dstar(K: int, sigma_target: float, k: int):
    """Direct dp_fill roofline sweep D* (SURVEY.md §8(d)): N_i = ceil(sigma^(1/K)) - 1,
    r_i = (k+i)*100, T = k^2*100.  Returns (counts, sizes, T)."""
    Ni = int(np.ceil(sigma_target ** (1.0 / K))) - 1
    counts = np.full(K, Ni, np.int32)
    sizes = np.array([(k + i) * 100 for i in range(K)], np.int64)
    return counts, sizes, k * k * 100
