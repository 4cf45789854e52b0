"""CG solve benchmark: (m^2 - D_eo D_oe) x = b on a 32^4 lattice, fp64.

python tools/bench_cg.py [--dims 32,32,32,32] [--mass 0.05] [--tol 1e-10] [--precision f64|mixed]
                        [--solver cg|mixed-cg --inner-tol 1e-4] [--force-halo 8 --transport p2p --push]
(--solver mixed-cg: fp32 inner CG on fp32 links with fp64 defect correction, dslash_cg_mixed)
Prints one JSON line: iterations, solve time, time per iteration, Dslash GFLOP/s inside the solve
(2 applies of 1146 flop/site per iteration), true residual.
"""
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
ap.add_argument("--mass", type=float, default=0.05)
ap.add_argument("--tol", type=float, default=1e-10)
ap.add_argument("--precision", default="f64")
ap.add_argument("--kernel", default="dir2")
ap.add_argument("--solver", default="cg", choices=["cg", "mixed-cg"])
ap.add_argument("--inner-tol", type=float, default=1e-4)
ap.add_argument("--force-halo", type=int, default=0, help="self-halo directions (bit mu), one GPU")
ap.add_argument("--transport", default="nccl", choices=["nccl", "p2p"])
ap.add_argument("--push", action="store_true", help="producer push (P2P transport): faces stored by the producing kernels")
ap.add_argument("--recon", type=int, default=18, choices=[18, 12, 9])
a = ap.parse_args()
dims = tuple(int(v) for v in a.dims.split(","))
fat, lng = fieldgen.workload_links(dims)
D = Dslash(dims, precision=a.precision, kernel=a.kernel, force_halo=a.force_halo, transport=a.transport, push=a.push,
           recon=a.recon)
D.load_links(fat, lng)
b = torch.from_numpy(fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 0)).cuda()
x = D.empty_vector()
outer = None
if a.solver == "cg":
    D.cg(x, b, 0, a.mass, rel_tol=1e-3, max_iter=20)   # warm-up
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    ok, it, res = D.cg(x, b, 0, a.mass, rel_tol=a.tol, max_iter=5000)
else:
    D.cg_mixed(x, b, 0, a.mass, rel_tol=1e-3, inner_tol=0.5, max_iter=20)   # warm-up (builds fp32 links)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    ok, it, outer, res = D.cg_mixed(x, b, 0, a.mass, rel_tol=a.tol, inner_tol=a.inner_tol, max_iter=10000)
torch.cuda.synchronize()
el = time.perf_counter() - t0
vh = D.vh
print(json.dumps({"dims": dims, "precision": a.precision, "recon": a.recon, "force_halo": a.force_halo,
                  "transport": a.transport, "push": a.push, "solver": a.solver, "outer_corrections": outer,
                  "inner_tol": a.inner_tol if a.solver != "cg" else None, "mass": a.mass, "tol": a.tol, "converged": ok,
                  "iterations": it, "solve_s": round(el, 4), "ms_per_iteration": round(1e3 * el / max(it, 1), 4),
                  "dslash_gflops_in_solver": round(2 * FLOP_PER_SITE * vh * it / el / 1e9, 1),
                  "true_rel_residual": res}))
D.close()
