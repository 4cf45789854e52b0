"""Timing probe of the producer push (DSLASH_OPT_PUSH) on one GPU.

Times the normal operator A = m^2 - D_{p,1-p} D_{1-p,p} (two applies; with the push the first
apply's boundary kernel stores its output faces straight into the ghost bank of the second) with
CUDA events over back-to-back calls, for a t-halo through the P2P transport with neighbour = self
(`force_halo`), without and with the push, next to the halo-free operator.  Prints one JSON line
per configuration.  usage: python tools/probe_push.py [--reps 200]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import fieldgen  # noqa: E402
from paper_conf_sc_dufekgaad024_b200 import Dslash  # noqa: E402


def time_normal(D, reps, m=0.3):
    b = torch.from_numpy(fieldgen.vector_cb(D.global_dims, 5, 0)).cuda()
    outs = [D.empty_vector() for _ in range(2)]
    for i in range(5):
        D.normal_apply(outs[i & 1], b, 0, m)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for i in range(reps):
        D.normal_apply(outs[i & 1], b, 0, m)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def time_cg(D, m=0.05, tol=1e-8):
    b = torch.from_numpy(fieldgen.vector_cb(D.global_dims, 6, 0)).cuda()
    x = D.empty_vector()
    D.cg(x, b, 0, m, rel_tol=1e-2)  # warm-up
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    ok, it, res = D.cg(x, b, 0, m, rel_tol=tol, max_iter=2000)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / max(it, 1), it


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=200)
    ap.add_argument("--cg", action="store_true")
    ap.add_argument("--cg-matrix", action="store_true", help="CG ms/iteration over transport/push/PDL/overlap")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    if a.cg_matrix:
        import time
        for dims in ((32, 32, 32, 32), (48, 48, 48, 6)):
            fat, lng = fieldgen.workload_links(dims)
            for kw in ({}, {"force_halo": 8}, {"force_halo": 8, "transport": "p2p"},
                       {"force_halo": 8, "transport": "p2p", "push": True},
                       {"force_halo": 8, "transport": "p2p", "pdl": False},
                       {"force_halo": 8, "transport": "p2p", "push": True, "pdl": False},
                       {"force_halo": 8, "transport": "p2p", "overlap": "none"},
                       {"force_halo": 8, "transport": "p2p", "push": True, "overlap": "none"}):
                with Dslash(dims, **kw) as D:
                    D.load_links(fat, lng)
                    runs = [time_cg(D)[0] for _ in range(3)]
                    b = torch.from_numpy(fieldgen.vector_cb(dims, 5, 0)).cuda()
                    o = D.empty_vector()
                    torch.cuda.synchronize()
                    t0 = time.perf_counter()
                    for _ in range(20):
                        D.normal_apply(o, b, 0, 0.3)
                    host_us = (time.perf_counter() - t0) / 20 * 1e6
                    torch.cuda.synchronize()
                    print(json.dumps({"dims": dims, "kw": kw, "cg_ms_per_iter": [round(r, 4) for r in runs],
                                      "host_enqueue_us_per_normal_apply": round(host_us, 1)}), flush=True)
            del fat, lng
        return
    cases = [((32, 32, 32, 32), 0x8), ((48, 48, 48, 6), 0x8), ((32, 32, 32, 32), 0xC)]
    for dims, mask in cases:
        fat, lng = fieldgen.workload_links(dims)
        rows = []
        for name, kw in (("no halo", {}), ("self-halo p2p", {"force_halo": mask, "transport": "p2p"}),
                         ("self-halo p2p + push", {"force_halo": mask, "transport": "p2p", "push": True})):
            with Dslash(dims, **kw) as D:
                D.load_links(fat, lng)
                ms = time_normal(D, a.reps)
                row = {"dims": dims, "halo_mask": mask, "mode": name, "normal_apply_ms": round(ms, 4),
                       "per_dslash_us": round(ms * 500, 1)}
                if a.cg:
                    ms_it, it = time_cg(D)
                    row.update(cg_ms_per_iter=round(ms_it, 4), cg_iters=it)
                rows.append(row)
                print(json.dumps(row), flush=True)
        del fat, lng


if __name__ == "__main__":
    main()
