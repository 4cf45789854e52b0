"""Launch-configuration sweep of the Dslash kernels (tuning aid; not the bench).

python tools/sweep.py [--dims 32,32,32,32] [--kernels site,dir4] [--blocks 64,128,256] [--steps 500]
Prints one JSON line per (kernel, block): us per apply, algorithmic GB/s, GFLOP/s.
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

import fieldgen
from paper_conf_sc_dufekgaad024_b200 import ALGO_BYTES, FLOP_PER_SITE, Dslash, _abi

ap = argparse.ArgumentParser()
ap.add_argument("--dims", default="32,32,32,32")
ap.add_argument("--kernels", default="site,dir2,dir4")
ap.add_argument("--blocks", default="64,128,256")
ap.add_argument("--minb", default="2,3,4")
ap.add_argument("--steps", type=int, default=500)
ap.add_argument("--halo", type=int, default=0)
ap.add_argument("--precision", default="f64")
ap.add_argument("--kernel-events", action="store_true", help="per-kernel events (cost ~3%%, block PDL overlap)")
ap.add_argument("--no-pdl", action="store_true")
a = ap.parse_args()
dims = tuple(int(v) for v in a.dims.split(","))
fat, lng = fieldgen.workload_links(dims)
l2 = torch.cuda.get_device_properties(0).L2_cache_size
for kern in a.kernels.split(","):
    D = Dslash(dims, parity_mask=0, kernel=kern, force_halo=a.halo, timing=a.kernel_events, precision=a.precision,
               pdl=not a.no_pdl)
    D.load_links(fat, lng)
    vb = 3 * D.vh * 16
    R = max(2, int(np.ceil(2 * l2 / (2 * vb))) + 1)
    srcs = [torch.from_numpy(fieldgen.vector_cb(dims, 3 + r, 1)).to(D.dtype).cuda() for r in range(R)]
    outs = [D.empty_vector() for _ in range(R)]
    for bs, mb in [(int(b), int(m)) for b in a.blocks.split(",") for m in a.minb.split(",")]:
        try:
            _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_BLOCK, bs)
            _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_MIN_BLOCKS, mb)
        except _abi.DslashError:
            continue
        for i in range(20):
            D.apply(outs[i % R], srcs[i % R], 0)
        torch.cuda.synchronize()
        D.kernel_timing_reset()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for i in range(a.steps):
            D.apply(outs[i % R], srcs[i % R], 0)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / a.steps
        kms, n = D.kernel_timing() if a.kernel_events else (ms * a.steps, a.steps)
        D.kernel_timing_reset()
        print(json.dumps({"dims": dims, "kernel": kern, "block": bs, "minb": mb, "us_per_apply": round(ms * 1e3, 2),
                          "kernel_us": round(kms / max(n, 1) * 1e3, 2),
                          "precision": a.precision, "algo_gbs": round(ALGO_BYTES[a.precision] * D.vh / (ms * 1e-3) / 1e9, 1),
                          "gflops": round(FLOP_PER_SITE * D.vh / (ms * 1e-3) / 1e9, 1)}), flush=True)
    D.close()
