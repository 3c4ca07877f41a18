"""K = 3 random dp_fill cases vs the oracle (ring-kernel debugging)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle
import paper_conf_ipps_ligsg18_b200 as P
rng = np.random.default_rng(1003)
bad = 0
for it in range(int(sys.argv[1]) if len(sys.argv) > 1 else 10):
    N = rng.integers(0, 26, 3).astype(np.int32)
    r = rng.integers(20, 200, 3).astype(np.int64)
    T = int(rng.integers(int(r.max()), int(r.max()) * 6))
    try:
        opt, tab, st = P.dp_fill(N, r, T)
    except Exception as e:
        print("FAIL", N.tolist(), r.tolist(), T, e, flush=True)
        raise
    want, _ = oracle.dp(N, r, T)
    ok = (tab.astype(np.int64) == want).all()
    bad += not ok
    print(N.tolist(), r.tolist(), T, "ok" if ok else "MISMATCH", flush=True)
print("bad", bad)
