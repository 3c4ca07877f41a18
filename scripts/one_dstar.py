"""One dp_fill of a D* geometry (for ncu launch lists): python scripts/one_dstar.py K sigma k"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_ligsg18_b200 as P
from synth import dstar
K, st, k = int(sys.argv[1]), float(sys.argv[2]), int(sys.argv[3])
N, r, T = dstar(K, st, k)
sg, e = P.dp_table_shape(N)
tab = torch.empty(sg * e, dtype=torch.uint8, device="cuda")
print(P.dp_fill_device(N, r, T, tab))
torch.cuda.synchronize()
