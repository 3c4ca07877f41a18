"""compute-sanitizer over the fill kernels (memcheck; racecheck on the split
mode's shared-memory reduction, the dataflow kernel's block ticket, and the
K = 3 cluster ring kernel's shared-memory ring with its DSMEM halo stores).  Small geometries that exercise every lane
layout: group widths that do not divide 32 (idle lanes), multi-word shifts
(GEN path), vector chunks CH = 1/2/4/8, uint8 and uint16 tables, split mode.
Parity of the same cases is checked in test_gpu_parity.py; here only memory
safety is asserted (exit code and the sanitizer's error summary).

Opt-in (PTAS_SANITIZER=1): the GPU pool this suite runs on has closed
compute-sanitizer (its wrapper refuses every run), so by default these tests
skip instead of invoking it.  Memory safety on the default path is covered by
the engine's own bounds checks (enumeration overflow flags, ETOOBIG guards)
and by the element-by-element parity tests.
"""
from __future__ import annotations

import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r"""
import sys
sys.path.insert(0, %(root)r)
import numpy as np
import paper_conf_ipps_ligsg18_b200 as P
cases = [
    ([3, 4, 18], [35, 50, 21], 110),          # W = 19: 5 words, Lg = 5 (2 idle lanes)
    ([2, 3, 4, 30], [40, 50, 60, 9], 150),    # W = 31 -> 8 words, CH = 2
    ([4, 5, 70], [90, 70, 11], 200),          # J0 > 4: multi-word shifts
    ([2, 2, 130], [60, 70, 9], 140),          # 36 words: CH = 2, Lg = 18
    ([2, 300], [60, 13], 120),                # uint16, 151 words: CH = 8
    ([1, 1, 1, 1, 1, 1, 40], [30, 31, 32, 33, 34, 35, 9], 120),
    ([6, 260], [40, 7], 100),                 # uint16, J0 > 2
    ([2, 700], [60, 13], 120),                # rows > 1 KiB: long-row path (row_cross + row_chain)
    ([6, 1500], [100, 99], 250),              # long rows, J0 = 2, ragged last chunk
]
for N, r, T in cases:
    P.dp_fill(np.array(N, np.int32), np.array(r, np.int64), T)
p = np.random.default_rng(0).integers(1, 100, 12)
P.ptas_solve(p, 3, 0.3)
# level window (VMM ring, slab launches), the K = 3 cluster ring kernel on a
# multi-CTA block, and the paper's Alg 4 partitioned A/B
for N, r, T in [([5, 4, 18], [35, 50, 21], 110), ([3, 3, 3, 30], [40, 50, 60, 9], 150), ([4, 300], [60, 13], 120)]:
    P.dp_fill_opt(np.array(N, np.int32), np.array(r, np.int64), T, window=1)
P.dp_fill(np.array([40, 30, 25], np.int32), np.array([700, 600, 500], np.int64), 1900)
P.dp_fill_alg4(np.array([5, 5, 5], np.int32), np.array([30, 40, 50], np.int64), 120, dim=3)
print("ok")
"""


def _run(tool, extra_env=None, timeout=900):
    if os.environ.get("PTAS_SANITIZER") != "1":
        pytest.skip("compute-sanitizer runs are opt-in (PTAS_SANITIZER=1): closed on the GPU pool")
    cs = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"
    if not os.path.exists(cs):
        pytest.skip("compute-sanitizer not found")
    env = dict(os.environ)
    env.update(extra_env or {})
    r = subprocess.run([cs, "--tool", tool, "--error-exitcode", "3", sys.executable, "-c", SCRIPT % {"root": ROOT}],
                       capture_output=True, text=True, timeout=timeout, env=env)
    out = r.stdout + r.stderr
    if "closed on this pool" in out:
        pytest.skip("compute-sanitizer is closed on this GPU pool")
    assert r.returncode == 0, out[-4000:]
    assert "ok" in r.stdout
    # memcheck: "ERROR SUMMARY: 0 errors"; racecheck: "RACECHECK SUMMARY: 0 hazards displayed (0 errors, 0 warnings)"
    assert "ERROR SUMMARY: 0 errors" in out or "(0 errors, 0 warnings)" in out, out[-4000:]


@pytest.mark.timeout(1200)
@pytest.mark.parametrize("env", [{"PTAS_DOMTAB": "1"}, {"PTAS_NC_CAP": "5"}, {"PTAS_NP_CAP": "2"}])
def test_memcheck_domtab_and_round_trip_free_enumeration(env):
    # dominance table forced for every geometry (D10); enumeration
    # bounds forced below |C| / the prefix count (D9: kernels exit, DP redone)
    _run("memcheck", env)


@pytest.mark.timeout(1200)
def test_memcheck_fill_layouts():
    _run("memcheck")


@pytest.mark.timeout(1200)
def test_memcheck_split_mode_and_forced_chunks():
    _run("memcheck", {"PTAS_SPLIT_ROWS": "1000000000", "PTAS_SWAR_CH": "2", "PTAS_DF": "0"})


@pytest.mark.timeout(1800)
def test_racecheck_split_mode():
    _run("racecheck", {"PTAS_SPLIT_ROWS": "1000000000", "PTAS_DF": "0"})


# dataflow launches (D7): warp row sets, block row sets (shared-memory ticket), mixed runs
@pytest.mark.timeout(1200)
@pytest.mark.parametrize("env", [{"PTAS_DF": "1"}, {"PTAS_DF": "3", "PTAS_DF_SPLIT_ROWS": "1000000000"},
                                 {"PTAS_DF": "3", "PTAS_DF_SPLIT_ROWS": "3"}])
def test_memcheck_dataflow(env):
    _run("memcheck", env)


@pytest.mark.timeout(1800)
def test_racecheck_dataflow_split():
    _run("racecheck", {"PTAS_DF": "3", "PTAS_DF_SPLIT_ROWS": "1000000000"})


@pytest.mark.timeout(1800)
def test_racecheck_default_paths():
    # default schedule: dataflow runs, per-level launches, the ring kernel (K = 3)
    _run("racecheck")


@pytest.mark.timeout(1200)
@pytest.mark.parametrize("tool", ["memcheck", "racecheck"])
def test_sanitizer_long_row_path_forced(tool):
    # the long-row two-launch path on every level of every case (PTAS_FORCE_SCALAR=2)
    _run(tool, {"PTAS_FORCE_SCALAR": "2"})
