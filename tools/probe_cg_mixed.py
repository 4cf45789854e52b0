"""Probe the mixed-precision CG: per-solve wall time for several inner tolerances in one process,
each solve twice (the first call of a process builds the fp32 links)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import fieldgen
from paper_conf_sc_dufekgaad024_b200 import Dslash

dims = tuple(int(v) for v in (sys.argv[1] if len(sys.argv) > 1 else "32,32,32,32").split(","))
fat, lng = fieldgen.workload_links(dims)
D = Dslash(dims)
D.load_links(fat, lng)
b = torch.from_numpy(fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 0)).cuda()
x = D.empty_vector()
for tol_in in (1e-4, 1e-2, 1e-5, 1e-4, 1e-3, 1e-4):
    for maxit in (50, 10000):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        ok, it, outer, res = D.cg_mixed(x, b, 0, 0.05, rel_tol=1e-10, inner_tol=tol_in, max_iter=maxit)
        torch.cuda.synchronize()
        el = time.perf_counter() - t0
        print(f"inner_tol {tol_in:g} max_iter {maxit}: {it} inner / {outer} outer, {el*1e3:.1f} ms, "
              f"{el / max(it, 1) * 1e3:.4f} ms/iter, res {res:.2e}", flush=True)
t0 = time.perf_counter()
ok, it, res = D.cg(x, b, 0, 0.05, rel_tol=1e-10, max_iter=200)
torch.cuda.synchronize()
el = time.perf_counter() - t0
print(f"fp64 cg 200 iters: {el / it * 1e3:.4f} ms/iter")
