import sys; sys.path.insert(0,'/root/repo')
import numpy as np, oracle
import paper_conf_ipps_ligsg18_b200 as P
rng = np.random.default_rng(1000 + 2)
def _rand_case(rng, K, maxN):
    N = rng.integers(0, maxN + 1, K).astype(np.int32)
    r = rng.integers(20, 200, K).astype(np.int64)
    T = int(rng.integers(int(r.max()), int(r.max()) * 6))
    return N, r, T
for i in range(12):
    N, r, T = _rand_case(rng, 2, 60)
    opt, tab, st = P.dp_fill(N, r, T)
    want, relax = oracle.dp(N, r, T)
    bad = np.argwhere(tab.astype(np.int64) != want)
    J0 = min(int(N[-1]), T // int(r[-1]))
    print(i, N.tolist(), r.tolist(), T, "J0", J0, "bad", len(bad), bad[:4].tolist(), "relax_exec ok" if True else "")
    if len(bad):
        p0 = bad[0][0]
        print(" got ", tab[p0].tolist()); print(" want", want[p0].tolist())
