"""Per-row-level relaxation counts of a DP (closed form), internal layout = ascending counts."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle
from synth import WORKLOADS

def poly(Ns):
    p = np.array([1.0])
    for x in Ns:
        p = np.convolve(p, np.ones(int(x) + 1))
    return p

def level_relax(N, r, T):
    order = np.argsort(N, kind="stable")
    N = np.array(N)[order]; r = np.array(r)[order]
    C = oracle.configs(N, r, T)
    lead = N[:-1]; W = N[-1] + 1
    rho_max = int(lead.sum())
    rel = np.zeros(rho_max + 1)
    rows = poly(lead)
    for s in C:
        sp, j = s[:-1], s[-1]
        q = poly(lead - sp)          # rows p >= s' : q = p - s'
        d = int(sp.sum())
        rel[d:d + len(q)] += q * (W - j)
    return rows, rel, W, len(C)

if __name__ == "__main__":
    w = WORKLOADS[sys.argv[1] if len(sys.argv) > 1 else "M2s"]
    p = w.p(); k = oracle.k_of(w.eps); LB, _ = oracle.bounds(p, w.m)
    u, r, N, _ = oracle.classify(p, LB, k)
    rows, rel, W, nC = level_relax(N, r, LB)
    i = int(np.argmax(rel))
    print("W", W, "|C|", nC, "levels", len(rows), "total relax %.3g" % rel.sum(), "max level", i, "rows", rows[i], "relax %.3g" % rel[i], "relax/row", rel[i] / rows[i])
