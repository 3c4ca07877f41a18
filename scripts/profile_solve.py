"""One M2s-style solve for ncu (no timing printed; a number under ncu is never a bench value)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_ligsg18_b200 as P  # noqa: E402
from synth import WORKLOADS  # noqa: E402

w = WORKLOADS[os.environ.get("WL", "M2s")]
torch.cuda.set_device(0)
reps = int(os.environ.get("REPS", "1"))
for _ in range(reps):
    r = P.ptas_solve(w.p(), w.m, w.eps, P=1, log=False)
print("launches/solve", r["stats"]["kernel_launches"], "fill", r["stats"]["fill_launches"], file=sys.stderr)
