"""Pinned host <-> device copy bandwidth on this box, the ceiling of bench.py's e2e number.

Per step the e2e path moves psi host->device and chi device->host (25.2 MB each at 32^4 fp64).
Measured with CUDA events over 200 copies of that size: H2D alone, D2H alone, and both at once
on two streams (full duplex), which is what dslash_apply_host_batch overlaps."""
import json
import sys

import torch


def main(nbytes=25165824, reps=200):
    torch.cuda.set_device(0)
    n = nbytes // 16
    h_in = [torch.empty(n, dtype=torch.complex128).pin_memory() for _ in range(4)]
    h_out = [torch.empty(n, dtype=torch.complex128).pin_memory() for _ in range(4)]
    d = [torch.empty(n, dtype=torch.complex128, device="cuda") for _ in range(8)]
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

    def timed(fn):
        fn(10)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn(reps)
        for s in (s1, s2):
            torch.cuda.current_stream().wait_stream(s)
        b.record()
        torch.cuda.synchronize()
        return a.elapsed_time(b) * 1e-3

    def h2d(k):
        s1.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s1):
            for i in range(k):
                d[i % 4].copy_(h_in[i % 4], non_blocking=True)

    def d2h(k):
        s2.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s2):
            for i in range(k):
                h_out[i % 4].copy_(d[4 + i % 4], non_blocking=True)

    t_h2d = timed(h2d)
    t_d2h = timed(d2h)
    t_both = timed(lambda k: (h2d(k), d2h(k)))
    res = {"bytes_per_copy": nbytes, "copies": reps,
           "h2d_gbs": round(nbytes * reps / t_h2d / 1e9, 2),
           "d2h_gbs": round(nbytes * reps / t_d2h / 1e9, 2),
           "duplex_gbs_each_way": round(nbytes * reps / t_both / 1e9, 2),
           "duplex_ms_per_pair": round(t_both / reps * 1e3, 4)}
    print(json.dumps(res))


if __name__ == "__main__":
    main(*(int(a) for a in sys.argv[1:]))
