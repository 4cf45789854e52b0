"""Halo-overlap timeline without a system profiler ("overlap is shown with a
timeline, NCCL kernels concurrent with the interior kernel").

With DSLASH_OPT_TIMING the library records CUDA events around every stencil kernel and around the
halo exchange on its communication stream; dslash_timeline returns those intervals on one clock.
This runs applies with a forced self-halo (neighbour = this rank) through the three transports on
one GPU: NCCL send/recv through a one-rank communicator (the P = 2 message pattern), device copies,
and the P2P copy engines, for the weak-scaling volume 32^3 x 32 (t halo) and t + z.  For the last
applies it prints each interval relative to the apply's interior-kernel start and the fraction of
the exchange that ran while the interior kernel ran.
usage: python tools/timeline.py [--dims 32,32,32,32] [--applies 20]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import fieldgen  # noqa: E402
from paper_conf_sc_dufekgaad024_b200 import Dslash  # noqa: E402


def overlap(a, b):
    return max(0.0, min(a[1], b[1]) - max(a[0], b[0]))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--dims", default="32,32,32,32")
    ap.add_argument("--applies", type=int, default=20)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    dims = tuple(int(v) for v in a.dims.split(","))
    fat, lng = fieldgen.workload_links(dims)
    srcs = [torch.from_numpy(fieldgen.vector_cb(dims, 3 + r, 1)).cuda() for r in range(4)]
    for mask in (0x8, 0xC):
        for name, kw in (("nccl-self", {"self_nccl": True}), ("device-copy", {}), ("p2p", {"transport": "p2p"})):
            with Dslash(dims, parity_mask=0, force_halo=mask, timing=True, **kw) as D:
                D.load_links(fat, lng)
                outs = [D.empty_vector() for _ in range(4)]
                for i in range(10):
                    D.apply(outs[i % 4], srcs[i % 4], 0)
                torch.cuda.synchronize()
                D.kernel_timing_reset()
                for i in range(a.applies):
                    D.apply(outs[i % 4], srcs[i % 4], 0)
                torch.cuda.synchronize()
                tl = D.timeline()
            # group per apply: each apply records exchange, span, interior, boundary (in that order)
            applies, cur = [], {}
            for kind, s, e in tl:
                if kind == "exchange" and cur:
                    applies.append(cur)
                    cur = {}
                cur.setdefault(kind, []).append((s, e))
            if cur:
                applies.append(cur)
            fr, rows = [], []
            for ap_ in applies[-5:]:
                t0 = ap_["interior"][0][0]
                rel = {k: [(round((s - t0) * 1e3, 1), round((e - t0) * 1e3, 1)) for s, e in v] for k, v in ap_.items()}
                rows.append(rel)
                x = ap_["exchange"][0]
                fr.append(overlap(x, ap_["interior"][0]) / max(x[1] - x[0], 1e-9))
            last = rows[-1]
            print(json.dumps({"dims": dims, "halo_mask": mask, "transport": name,
                              "last_apply_us_rel_to_interior_start": last,
                              "exchange_fraction_under_interior": [round(f, 3) for f in fr]}), flush=True)


if __name__ == "__main__":
    main()
