"""Where the multi-RHS CG iteration goes (32^4, 8 systems, fp64): time 200 CG iterations, 400 blocked
8-RHS applies alone, with PDL on and off.  python tools/cg_multi_profile.py"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import fieldgen
from paper_conf_sc_dufekgaad024_b200 import Dslash

dims = (32, 32, 32, 32)
fat, lng = fieldgen.workload_links(dims)
for pdl in (True, False):
    D = Dslash(dims, kernel="site", pdl=pdl)
    D.load_links(fat, lng)
    planar = torch.stack([torch.from_numpy(fieldgen.vector_cb(dims, 5 + k, 0)) for k in range(8)]).contiguous().cuda()
    bb = D.to_blocked(torch.empty_like(planar), planar)
    xb, t = torch.empty_like(bb), torch.empty_like(bb)
    D.cg_multi_blocked(xb, bb, 0, 0.05, rel_tol=1e-30, max_iter=20)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    D.cg_multi_blocked(xb, bb, 0, 0.05, rel_tol=1e-30, max_iter=200)
    torch.cuda.synchronize()
    t_cg = (time.perf_counter() - t0) / 200
    for i in range(20):
        D.apply_multi_blocked(t, bb, 1)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for i in range(200):
        D.apply_multi_blocked(t, bb, 1)
        D.apply_multi_blocked(xb, t, 0)
    torch.cuda.synchronize()
    t_ap = (time.perf_counter() - t0) / 200
    print(f"pdl={pdl}: CG iteration {t_cg * 1e3:.3f} ms, two blocked applies {t_ap * 1e3:.3f} ms, rest {1e3 * (t_cg - t_ap):.3f} ms")
    D.close()
