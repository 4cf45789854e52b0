"""Multi-RHS CG benchmark: nrhs systems (m^2 - D_eo D_oe) x_r = b_r at 32^4, fp64, solved together by
dslash_cg_multi_blocked (every iteration = two 8-RHS site-blocked stencil passes) vs one after the
other by dslash_cg.  python tools/bench_cg_multi.py [--nrhs 8] [--mass 0.05] [--tol 1e-10]
Prints one JSON line."""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import fieldgen
from paper_conf_sc_dufekgaad024_b200 import FLOP_PER_SITE, Dslash

ap = argparse.ArgumentParser()
ap.add_argument("--dims", default="32,32,32,32")
ap.add_argument("--nrhs", type=int, default=8)
ap.add_argument("--mass", type=float, default=0.05)
ap.add_argument("--tol", type=float, default=1e-10)
ap.add_argument("--precision", default="f64", choices=["f64", "mixed"])
a = ap.parse_args()
dims = tuple(int(v) for v in a.dims.split(","))
fat, lng = fieldgen.workload_links(dims)
D = Dslash(dims, precision=a.precision, kernel="site")
D.load_links(fat, lng)
planar = torch.stack([torch.from_numpy(fieldgen.vector_cb(dims, fieldgen.SEED_PSI + k, 0))
                      for k in range(a.nrhs)]).contiguous().cuda()
bb = D.to_blocked(torch.empty_like(planar), planar)
xb = torch.empty_like(bb)
D.cg_multi_blocked(xb, bb, 0, a.mass, rel_tol=1e-3, max_iter=16)   # warm-up
torch.cuda.synchronize()
t0 = time.perf_counter()
ok, its, res = D.cg_multi_blocked(xb, bb, 0, a.mass, rel_tol=a.tol, max_iter=5000)
torch.cuda.synchronize()
t_multi = time.perf_counter() - t0
x = D.empty_vector()
D.cg(x, planar[0].contiguous(), 0, a.mass, rel_tol=1e-3, max_iter=16)  # warm-up
torch.cuda.synchronize()
t0 = time.perf_counter()
single = []
for k in range(a.nrhs):
    oks, it_k, res_k = D.cg(x, planar[k].contiguous(), 0, a.mass, rel_tol=a.tol, max_iter=5000)
    single.append((oks, it_k, res_k))
torch.cuda.synchronize()
t_single = time.perf_counter() - t0
vh = D.vh
it_max = max(its)
print(json.dumps({
    "what": f"{a.nrhs} systems, {a.precision}, {dims}, m={a.mass}, tol={a.tol}",
    "multi": {"converged": ok, "iterations": its, "true_rel_resid": [float(f"{r:.3g}") for r in res],
              "solve_s": round(t_multi, 4), "ms_per_iteration": round(1e3 * t_multi / it_max, 4),
              "dslash_tflops": round(2 * FLOP_PER_SITE * vh * a.nrhs * it_max / t_multi / 1e12, 2)},
    "one_by_one": {"converged": all(s[0] for s in single), "iterations": [s[1] for s in single],
                   "true_rel_resid": [float(f"{s[2]:.3g}") for s in single], "solve_s": round(t_single, 4)},
    "speedup": round(t_single / t_multi, 3)}))
