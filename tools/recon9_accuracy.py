"""Normwise error of the reduced-precision paths against the fp64 oracle, per long-link
compression (is the fp32 recon-9 rebuild's hardware sin/cos visible?).

    python tools/recon9_accuracy.py [L]   (default 16: an L^4 lattice, both parities)
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import fieldgen
import oracle
from paper_conf_sc_dufekgaad024_b200 import Dslash

L = int(sys.argv[1]) if len(sys.argv) > 1 else 16
dims = (L, L, L, L)
torch.cuda.set_device(0)
fat, lng = fieldgen.workload_links(dims)
psi = fieldgen.vector(dims, fieldgen.SEED_PSI)
refs = {p: oracle.full_to_cb(oracle.dslash(fat, lng, psi, p), p) for p in (0, 1)}
for precision in ("f64", "f32", "mixed"):
    errs = {}
    for recon in (18, 12, 9):
        e = 0.0
        with Dslash(dims, precision=precision, recon=recon, kernel="site" if recon == 9 else "dir2") as D:
            D.load_links(fat, lng)
            for p in (0, 1):
                src = torch.from_numpy(fieldgen.vector_cb(dims, fieldgen.SEED_PSI, 1 - p)).to(D.dtype).cuda()
                got = D(src, p).cpu().numpy().astype(np.complex128)
                e = max(e, oracle.normwise_error(got, refs[p]))
        errs[recon] = e
    print(f"{L}^4 {precision:6s} normwise error vs fp64 oracle: recon-18 {errs[18]:.3e}  recon-12 {errs[12]:.3e}  "
          f"recon-9 {errs[9]:.3e}  (recon-9 / recon-18 = {errs[9] / errs[18]:.2f})", flush=True)
