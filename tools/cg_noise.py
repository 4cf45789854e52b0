"""CG timing noise probe: repeated CG solves at 32^4, ms per iteration next to the stencil kernels'
own time inside each solve (per-kernel CUDA events, DSLASH_OPT_TIMING), so a slow solve can be
told apart as slower kernels (clocks, power) or gaps between them (launch / dependency stalls)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import fieldgen  # noqa: E402
from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi  # noqa: E402
from tools.probe_push import time_cg  # noqa: E402

torch.cuda.set_device(0)
dims = (32, 32, 32, 32)
fat, lng = fieldgen.workload_links(dims)
for kw in ({}, {"timing": True}, {"pdl": False}, {"force_halo": 8, "transport": "p2p", "push": True}):
    with Dslash(dims, **kw) as D:
        D.load_links(fat, lng)
        for r in range(6):
            if kw.get("timing"):
                D.kernel_timing_reset()
            t0 = time.perf_counter()
            ms, it = time_cg(D)
            row = {"kw": kw, "run": r, "ms_per_iter": round(ms, 4), "iters": it,
                   "wall_s": round(time.perf_counter() - t0, 3)}
            if kw.get("timing"):
                tot, n = D.kernel_timing(_abi.DSLASH_TIMING_INTERIOR)
                row.update(stencil_us_per_launch=round(tot / max(n, 1) * 1e3, 1), launches=n)
            print(json.dumps(row), flush=True)
