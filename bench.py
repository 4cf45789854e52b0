#!/usr/bin/env python
"""Benchmark of the single-parity HISQ Dslash (BASELINE.json metric: Dslash GFLOP/s and
achieved HBM GB/s, % of B200 peak, at 1/2/4/8 GPUs).

One step = one Dslash apply (every row of SURVEY.md §8(a): site decode, neighbour addressing,
link stream, neighbour gather, 16 matvecs, store; plus the depth-3 halo exchange when N > 1)
on one batch of synthetic fp64 input.

  N = 1 : 32^4 lattice (BASELINE.json configs[2], the paper's workload).
  N > 1 : weak scaling, 32^3 x 32N global lattice t-partitioned over N GPUs (configs[4] shape:
          32^3 x 32 per GPU), halo overlapped with the interior kernel.
  --global-dims 48,48,48,48 : strong scaling (configs[3]); the process grid is chosen by the
          rule in choose_grid() unless --grid is given.

GFLOP/s = 1146 flop x target sites / time (PAPER.md L278 convention, 600.8 MFLOP per 32^4
apply).  Algorithmic bytes = 2400 per target site.  Inputs are larger than L2:
the 1.2 GB of links stream through every apply and the source/output vectors rotate over R
pairs whose footprint exceeds the 126 MB L2.

Timing (CUDA events around back-to-back applies on one in-order stream): the
timed region holds exactly the applies, with no per-kernel events at any N (they cost ~3% and
block programmatic dependent launch); max over ranks.  The per-kernel breakdown behind
`roofline` (interior / boundary kernels, their span) comes from a separate pass after the timed
region whenever a step holds more than one launch.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--kernel site|dir2|dir4] [--block B]
  python bench.py --impl reference ...   # the CPU oracle on the host cores (reference arm)

Without torchrun, --gpus N > 1 launches itself under torch.distributed.run (one process per
GPU, 127.0.0.1 rendezvous); rank 0 prints the one JSON line either way.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

FLOP_PER_SITE = 1146
ALGO_BYTES_PER_SITE = 2400
METRIC = "Dslash GFLOP/s and achieved HBM GB/s (% of B200 peak) at 1/2/4/8 GPUs"
NOMINAL_HBM_GBS = 8000.0
FALLBACK_HBM_GBS = 6650.0  # /opt/skills/guides/B200_PROFILING.md fallback


def parse(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=2000)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--kernel", default=None, choices=["site", "dir2", "dir4"],
                    help="default: dir2 (site with --recon 9, --nrhs > 1 or --precision mixed, measured best for them)")
    ap.add_argument("--min-blocks", type=int, default=0)
    ap.add_argument("--layout", default="planar", choices=["planar", "blocked"],
                    help="multi-RHS vector layout: planar [nrhs][3][Vh] (dslash_apply_multi) or site-blocked "
                         "[Vh/16][nrhs*3][16] (dslash_apply_multi_blocked; no halo)")
    ap.add_argument("--nrhs", type=int, default=1, choices=[1, 2, 3, 4, 5, 6, 7, 8],
                    help="right-hand sides per apply, one link pass (SURVEY §8(f)-4)")
    ap.add_argument("--recon", type=int, default=18, choices=[18, 12, 9],
                    help="12: long links stored as 2 rows (SURVEY §8(f)-2, QUDA recon-12, PAPER.md L325); "
                         "9: 8 SU(3) parameters + a phase")
    ap.add_argument("--precision", default="f64", choices=["f64", "f32", "mixed"],
                    help="f64 is the paper's (L278) and the headline; f32/mixed are SURVEY §8(f)-1")
    ap.add_argument("--block", type=int, default=0)
    ap.add_argument("--local", default="32,32,32,32", help="per-GPU local extents x,y,z,t (weak scaling)")
    ap.add_argument("--global-dims", default=None,
                    help="strong scaling: fixed global lattice x,y,z,t (e.g. 48,48,48,48, configs[3])")
    ap.add_argument("--grid", default=None,
                    help="process grid x,y,z,t (default: 1,1,1,N for weak scaling; choose_grid() for strong)")
    ap.add_argument("--flush-l2", action="store_true",
                    help="write a 2x-L2 buffer between steps (for lattices whose links fit in L2, e.g. 16^4); "
                         "value then uses the summed kernel times, the flush excluded")
    ap.add_argument("--force-halo", type=int, default=0,
                    help="bitmask of directions run through the halo path with neighbour = self (1 GPU)")
    ap.add_argument("--parity", type=int, default=0)
    ap.add_argument("--no-overlap", action="store_true")
    ap.add_argument("--overlap", default="sites", choices=["sites", "dirs"],
                    help="with a halo: split by sites (interior box during the exchange, boundary slabs "
                         "after) or by direction (local hops of every site during the exchange, ghost hops "
                         "after)")
    ap.add_argument("--colocate", action="store_true",
                    help="testing aid: every rank on GPU 0 (gloo process group, P2P transport); checks the N > 1 "
                         "code path on a one-GPU box -- its timings are not scaling numbers")
    ap.add_argument("--stage", action="store_true",
                    help="neighbour-staged kernel: x/y source rows of a tile copied to shared memory by TMA "
                         "(site / dir2 variants)")
    ap.add_argument("--self-nccl", action="store_true",
                    help="with --force-halo at N = 1: self-neighbour faces through NCCL send/recv to this rank "
                         "(one-rank communicator; the P = 2 message pattern)")
    ap.add_argument("--transport", default="nccl", choices=["nccl", "p2p"],
                    help="halo transport for N > 1: NCCL send/recv, or copy-engine puts into IPC-mapped ghosts")
    ap.add_argument("--no-pdl", action="store_true",
                    help="ordinary launches instead of programmatic dependent launch (DSLASH_OPT_PDL)")
    ap.add_argument("--halo-dryrun", action="store_true",
                    help="timing aid: the exchange keeps its stream structure but moves no bytes (results WRONG)")
    ap.add_argument("--breakdown-steps", type=int, default=200,
                    help="steps of the separate per-kernel-event pass after the timed region (0: none)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-read-calibration", action="store_true",
                    help="skip the same-run HBM read-stream calibration (2 GiB torch.sum)")
    ap.add_argument("--cpu-seconds", type=float, default=12.0, help="oracle CPU-baseline budget")
    ap.add_argument("--no-oracle-48", action="store_true",
                    help="skip the 48^4 oracle leg of cpu_baseline (SURVEY §8(d): 32^4 and 48^4)")
    ap.add_argument("--selftest-launch", action="store_true",
                    help="CPU check of the launch contract only: ranks rendezvous over gloo, take the max "
                         "of a per-rank number and rank 0 prints one JSON line (no CUDA)")
    args = ap.parse_args(argv)
    if args.kernel is None:
        # measured per configuration (profiles/r03/recon_mapping_ab.txt, mapping_mixed_ab.txt): site for
        # recon-9, multi-RHS and mixed precision (mixed 96.2 vs 99.9 us, mixed recon-12 83.4 vs 88.6),
        # dir2 otherwise (fp64 / fp32: +1%)
        args.kernel = "site" if (args.recon == 9 or args.nrhs > 1 or args.precision == "mixed") else "dir2"
    return args


# --------------------------------------------------------------------------- decomposition
def interior_fraction(local, halo_dims):
    """Fraction of local sites whose 16 sources are all local (depth-3 halo in halo_dims)."""
    f = 1.0
    for d in halo_dims:
        f *= max(0, local[d] - 6) / local[d]
    return f


def choose_grid(gdims, n):
    """Strong-scaling process grid {1, 1, Pz, Pt} with Pz * Pt = n (north star:
    partition t first, then z).

    Rule: t alone while the local t extent keeps at least half the sites interior (Lt / n >= 12:
    a depth-3 face on each side of >= 6 interior slices); otherwise, among the grids whose
    partitioned local extents are even and >= 4 (depth-3 halo, parity), the one with the largest
    interior fraction (sites that compute while the faces are in flight), then the fewest face
    bytes, then the larger Pt (t-faces are contiguous: zero-copy sends).  48^4: t1, t2, t4, and on
    8 GPUs z2 x t4 (37.5% interior, 11.9 MB of faces per GPU) instead of t8 (local Lt = 6: no
    interior site, 15.9 MB).
    """
    if gdims[3] % n == 0 and (n == 1 or (gdims[3] // n >= 12 and (gdims[3] // n) % 2 == 0)):
        return (1, 1, 1, n)
    best = None
    for pz in range(1, n + 1):
        if n % pz:
            continue
        pt = n // pz
        grid = (1, 1, pz, pt)
        if any(g % p for g, p in zip(gdims, grid)):
            continue
        loc = [g // p for g, p in zip(gdims, grid)]
        halo = [d for d in (2, 3) if grid[d] > 1]
        if any(loc[d] < 4 or loc[d] % 2 for d in halo):
            continue
        vol = loc[0] * loc[1] * loc[2] * loc[3]
        face_bytes = sum(2 * 3 * (vol // loc[d]) // 2 * 48 for d in halo)
        key = (interior_fraction(loc, halo), -face_bytes, pt)
        if best is None or key > best[0]:
            best = (key, grid)
    if best is None:
        raise SystemExit(f"no valid z/t process grid for {gdims} on {n} GPUs")
    return best[1]


def workload(args, world):
    if args.global_dims:
        gdims = tuple(int(v) for v in args.global_dims.split(","))
        grid = tuple(int(v) for v in args.grid.split(",")) if args.grid else choose_grid(gdims, world)
        loc = tuple(g // p for g, p in zip(gdims, grid))
        name = (f"{gdims[0]}x{gdims[1]}x{gdims[2]}x{gdims[3]} fp64 single-parity HISQ Dslash, strong scaling, "
                f"grid {'x'.join(map(str, grid))} (configs[3] shape)")
        return gdims, grid, loc, name
    grid = tuple(int(v) for v in args.grid.split(",")) if args.grid else (1, 1, 1, world)
    loc = tuple(int(v) for v in args.local.split(","))
    gdims = tuple(l * p for l, p in zip(loc, grid))
    if world == 1 and loc == (32, 32, 32, 32):
        name = "32^4 fp64 single-parity HISQ Dslash, 1 GPU (BASELINE.json configs[2])"
    else:
        name = (f"{gdims[0]}^3x{gdims[3]} fp64 single-parity HISQ Dslash, weak scaling "
                f"{loc[0]}x{loc[1]}x{loc[2]}x{loc[3]} per GPU, t-partitioned over {world} (configs[4] shape)")
    return gdims, grid, loc, name


# --------------------------------------------------------------------------- records
def measured_peak():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            v = float(json.load(f)["hbm_gbs"])
            return v, "measured (MEASURED_PEAKS.json hbm_gbs, copy burst)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


def ncu_traffic(kernel_name, local_dims):
    """dram read+write bytes per launch from the committed ncu --set full summary, if it matches."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_summary.json")) as f:
            s = json.load(f)
        for e in s.get("kernels", []):
            if e.get("variant") == kernel_name and tuple(e.get("local_dims", ())) == tuple(local_dims):
                return int(e["dram_bytes_per_launch"])
    except Exception:
        pass
    return None


class ClockSampler:
    """Samples SM clock and throttle reasons with NVML from the start of the warm-up to the end of
    the timed region.  The polling thread starts (and makes its first, slow NVML calls) before
    the window opens; inside the window it records a sample every ~0.1 ms and the interpreter
    switches threads every 50 us, so even a 20-step run (~5 ms of GPU work) gets >= 10 samples."""

    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}
    PERIOD_S = 0.0001

    def __init__(self, device_index):
        self.samples, self.reasons, self.max_mhz = [], 0, None
        self._stop = threading.Event()
        self._active = threading.Event()
        self.t_start = self.t_stop = None
        self._switch = sys.getswitchinterval()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.hdl = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.hdl, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None
        if self.nv:
            self._ready = threading.Event()
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
            self._ready.wait(5.0)

    def _sample(self):
        c = self.nv.nvmlDeviceGetClockInfo(self.hdl, self.nv.NVML_CLOCK_SM)
        r = int(self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.hdl))
        return c, r

    def _run(self):
        try:
            self._sample()          # first calls (lazy NVML setup) outside the window
        except Exception:
            pass
        self._ready.set()
        while not self._stop.is_set():
            if not self._active.wait(0.001):
                continue
            try:
                c, r = self._sample()
                if self._active.is_set():
                    self.samples.append(c)
                    self.reasons |= r
            except Exception:
                pass
            time.sleep(self.PERIOD_S)

    def start(self):
        sys.setswitchinterval(5e-5)
        self.t_start = time.perf_counter()
        self._active.set()
        return self

    def stop(self):
        self._active.clear()
        self.t_stop = time.perf_counter()
        sys.setswitchinterval(self._switch)
        self._stop.set()
        if self.nv:
            self.t.join()

    def summary(self):
        window = round((self.t_stop - self.t_start) * 1e3, 2) if self.t_stop else None
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["unavailable"], "samples": 0}
        s = sorted(self.samples)
        names = [n for b, n in self.REASONS.items() if self.reasons & b and n != "gpu_idle"]
        return {"sm_mhz": s[len(s) // 2], "sm_max_mhz": self.max_mhz, "sm_min_mhz": s[0], "reasons": names,
                "samples": len(s), "window": "warm-up start to timed-region end", "window_ms": window}


def host_cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count()


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


# --------------------------------------------------------------------------- the CPU oracle legs
def run_oracle_baseline(gdims, parity, budget_s, steps=None, warmup=0):
    """Time the CPU oracle (as it stands) on the host cores.  Returns (cpu_baseline dict, s/step).

    steps=None: full-lattice applies until `budget_s` is spent (>= 1), plus one single-threaded
    apply.  steps=K: the reference arm, K timed steps after `warmup`, each a bounded sample of
    target sites sized so the whole run takes about `budget_s`.
    """
    import numpy as np

    import fieldgen
    import oracle

    fat, lng = fieldgen.workload_links(gdims)
    psi = fieldgen.vector(gdims, fieldgen.SEED_PSI)
    vh = int(np.prod(gdims)) // 2
    cores = host_cores()
    tag = f"{gdims[0]}x{gdims[1]}x{gdims[2]}x{gdims[3]}"
    t0 = time.perf_counter()
    oracle.dslash(fat, lng, psi, parity, cores)                 # warm-up full apply
    t_full = time.perf_counter() - t0
    if steps is None:
        n, t0 = 0, time.perf_counter()
        while True:
            oracle.dslash(fat, lng, psi, parity, cores)
            n += 1
            el = time.perf_counter() - t0
            if el >= budget_s:
                break
        t0 = time.perf_counter()
        oracle.dslash(fat, lng, psi, parity, 1)                  # one single-threaded apply
        t1 = time.perf_counter() - t0
        return {"value": FLOP_PER_SITE * vh * n / el / 1e9, "unit": "GFLOP/s", "cores": cores,
                "kind": "oracle", "cpu": cpu_model(), "lattice": list(gdims),
                "value_1_thread": FLOP_PER_SITE * vh / t1 / 1e9,
                "sample": f"{n} full {tag} applies (parity {parity}), {el:.1f} s, OpenMP over target sites; "
                          f"value_1_thread: one apply on 1 thread"}, el / n
    sites_all = oracle.lex_sites_of_parity(gdims, parity)
    frac = min(1.0, budget_s / max(1, steps + warmup) / t_full)
    stride = max(1, int(round(1.0 / frac)))
    sites = np.ascontiguousarray(sites_all[::stride])
    for _ in range(warmup):
        oracle.dslash_sites(fat, lng, psi, sites, cores)
    t0 = time.perf_counter()
    for _ in range(steps):
        oracle.dslash_sites(fat, lng, psi, sites, cores)
    el = time.perf_counter() - t0
    return {"value": FLOP_PER_SITE * sites.size * steps / el / 1e9, "unit": "GFLOP/s", "cores": cores,
            "kind": "oracle", "cpu": cpu_model(), "lattice": list(gdims),
            "sample": f"each step: every {stride}-th target site of the {tag} lattice ({sites.size} of {vh} "
                      f"sites), parity {parity}"}, el / steps


def oracle_leg(gdims, parity, budget_s):
    """One extra oracle timing (the oracle at 32^4 AND 48^4, on 1 thread and on all
    cores): a compact record for cpu_baseline["legs"]."""
    cb, _ = run_oracle_baseline(gdims, parity, budget_s)
    return {k: cb[k] for k in ("lattice", "value", "value_1_thread", "cores", "sample")}


def reference_arm(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    world = args.gpus
    gdims, grid, loc, name = workload(args, 1)   # the oracle runs the N=1 workload of one rank
    budget = max(20.0, min(150.0, 0.05 * (args.steps + args.warmup)))
    cb, per_step = run_oracle_baseline(gdims, args.parity, budget, args.steps, args.warmup)
    line = {"metric": METRIC, "value": cb["value"], "unit": "GFLOP/s", "impl": "reference", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": per_step * 1e3, "higher_is_better": True,
            "scaling": "strong" if args.global_dims else "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": name, "global_dims": list(gdims), "parity": args.parity,
                       "oracle": "oracle/hisq_oracle.c (plain C99 complex, -O2 -ffp-contract=off, OpenMP)"},
            "cpu_baseline": cb,
            "e2e": {"value": cb["value"], "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# --------------------------------------------------------------------------- launch
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def self_launch(args):
    """--gpus N > 1 outside torchrun: run this script under torch.distributed.run, one process
    per GPU on this node (127.0.0.1 rendezvous).  Rank 0's JSON line reaches our stdout."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={_free_port()}", os.path.abspath(__file__), *sys.argv[1:]]
    env = dict(os.environ)
    env.setdefault("OMP_NUM_THREADS", "1")
    return subprocess.run(cmd, env=env).returncode


def selftest_launch(args):
    """The launch contract without a GPU: rendezvous, barrier, max over ranks, one JSON line."""
    import torch
    import torch.distributed as dist
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if world > 1:
        dist.init_process_group("gloo")
        dist.barrier()
    t = torch.tensor([float(rank + 1)], dtype=torch.float64)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    if rank == 0:
        print(json.dumps({"selftest_launch": True, "n_gpus": args.gpus, "world_size": world,
                          "max_over_ranks": float(t.item())}), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return self_launch(args)
    if args.selftest_launch:
        return selftest_launch(args)
    if args.impl == "reference":
        return reference_arm(args)
    # The bench's stdout is the one JSON line.  Native code may print to fd 1 (NCCL prints its
    # "NCCL version" banner with printf at communicator init when NCCL_DEBUG is set), so fd 1
    # points at stderr for the whole run and is restored only for the JSON line.
    sys.stdout.flush()
    real_stdout = os.dup(1)
    os.dup2(2, 1)

    import numpy as np
    import torch
    import torch.distributed as dist

    import fieldgen
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi, algo_bytes

    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.gpus != world:
        os.dup2(real_stdout, 1)
        print(json.dumps({"error": f"--gpus {args.gpus} but WORLD_SIZE {world}"}))
        return 2
    if args.colocate:
        local_rank = 0
        args.transport = "p2p"
    torch.cuda.set_device(local_rank)
    if world > 1:
        if args.colocate:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    gdims, grid, loc, name = workload(args, world)
    parity = args.parity

    nrhs = args.nrhs
    algo_bytes_site = algo_bytes(args.precision, args.recon, nrhs)
    D = Dslash(gdims, grid, parity_mask=parity, kernel=args.kernel, block=args.block, min_blocks=args.min_blocks,
               timing=bool(args.flush_l2), precision=args.precision, recon=args.recon,
               overlap="none" if args.no_overlap else args.overlap, rank=rank, world_size=world,
               force_halo=args.force_halo, pdl=not args.no_pdl,
               transport=args.transport if world > 1 or args.force_halo else "nccl",
               self_nccl=bool(args.self_nccl and world == 1 and args.force_halo and args.transport == "nccl"),
               stage=args.stage)
    if args.halo_dryrun:
        _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_HALO_DRYRUN, 1)
    origin, extent = D.origin, D.local_dims
    fat, lng = fieldgen.workload_links(gdims, origin=origin, extent=extent)
    D.load_links(fat, lng)
    del fat, lng
    vh = D.vh
    plan = D.plan
    halo = any(plan.halo)
    vec_bytes = 3 * vh * (8 if args.precision == "f32" else 16) * nrhs   # one step's source (or output)
    l2_bytes = torch.cuda.get_device_properties(torch.cuda.current_device()).L2_cache_size
    R = max(2, int(np.ceil(2 * l2_bytes / (2 * vec_bytes))) + 1)

    def make_src(r):
        vs = [torch.from_numpy(fieldgen.vector_cb(gdims, fieldgen.SEED_PSI + r * nrhs + k, 1 - parity, origin=origin,
                                                  extent=extent)).to(D.dtype) for k in range(nrhs)]
        return (vs[0] if nrhs == 1 else torch.stack(vs)).contiguous()

    srcs = [make_src(r).cuda() for r in range(R)]
    if args.layout == "blocked":   # converted once, on the device, before the timed region
        srcs = [D.to_blocked(torch.empty_like(v), v) for v in srcs]
    outs = [torch.empty_like(srcs[0]) for _ in range(R)]
    stream = torch.cuda.current_stream()
    flush = torch.empty(2 * l2_bytes // 4, dtype=torch.float32, device="cuda") if args.flush_l2 else None
    red_dev = "cpu" if args.colocate else "cuda"

    def step(i):
        if flush is not None:
            flush.fill_(float(i))
        if args.layout == "blocked":
            D.apply_multi_blocked(outs[i % R], srcs[i % R], parity, stream)
        elif nrhs == 1:
            D.apply(outs[i % R], srcs[i % R], parity, stream)
        else:
            D.apply_multi(outs[i % R], srcs[i % R], parity, stream)

    def max_over_ranks(v):
        t = torch.tensor([v], dtype=torch.float64, device=red_dev)
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    # ---- warm-up + timed region (no per-kernel events unless --flush-l2, whose flush writes are
    # not Dslash work and must be excluded)
    clk = ClockSampler(torch.cuda.current_device()).start()
    for i in range(args.warmup):
        step(i)
    torch.cuda.synchronize()
    D.kernel_timing_reset()   # discard warm-up records
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    ev0.record(stream)
    for i in range(args.steps):
        step(i)
    ev1.record(stream)
    torch.cuda.synchronize()
    clk.stop()
    if world > 1:
        dist.barrier()
    ms = ev0.elapsed_time(ev1)
    if args.flush_l2:
        ms = D.kernel_timing(_abi.DSLASH_TIMING_ALL)[0]
        D.kernel_timing_reset()
    ms_max = max_over_ranks(ms)
    total_sites = vh * world * nrhs      # site-RHS pairs per step
    gflops = FLOP_PER_SITE * total_sites * args.steps / (ms_max * 1e-3) / 1e9
    algo_gbs = algo_bytes_site * vh * world * args.steps / (ms_max * 1e-3) / 1e9

    # ---- dominant-kernel record.  One stencil launch per step (no halo): the timed region's
    # events / launches ARE the average launch duration (launch gaps included).  Several launches
    # per step (halo): a separate pass with per-kernel events, after the timed region.
    peak, peak_src = measured_peak()
    lanes_n = {"site": 1, "dir2": 2, "dir4": 4}[args.kernel]
    kstem = "dslash_stage_kernel" if args.stage else "dslash_kernel"
    breakdown = None
    launches_per_step = 1
    if not halo:
        kern_ms, n_launch, dom_sites = ms_max / args.steps, args.steps, vh
        kname = (f"{kstem}<lanes={lanes_n}, ghost=false> (all sites): duration = CUDA events around the timed "
                 f"region / launches (1 stencil launch per step{', PDL' if not args.no_pdl else ''})")
        if args.flush_l2:
            kname = f"{kstem}<lanes={lanes_n}, ghost=false> (all sites): per-launch CUDA events (L2 flushed between steps)"
    else:
        nb = max(1, args.breakdown_steps)
        _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_TIMING, 1)
        for i in range(nb):
            step(i)
        torch.cuda.synchronize()
        t_int, n_int = D.kernel_timing(_abi.DSLASH_TIMING_INTERIOR)
        t_bnd, n_bnd = D.kernel_timing(_abi.DSLASH_TIMING_BOUNDARY)
        t_all, n_all = D.kernel_timing(_abi.DSLASH_TIMING_ALL)
        t_span, n_span = D.kernel_timing(_abi.DSLASH_TIMING_SPAN)
        t_x, n_x = D.kernel_timing(_abi.DSLASH_TIMING_EXCHANGE)
        D.kernel_timing_reset()
        _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_TIMING, 0)
        launches_per_step = max(1, n_all // nb)
        if n_span:              # interior and boundary overlap: their span is the apply's stencil time
            kern_ms, n_launch = max_over_ranks(t_span / n_span), n_span
            kname = (f"{kstem}<lanes={lanes_n}> interior + boundary ("
                     + ("local pass + ghost pass, split by direction" if args.overlap == "dirs" else
                        "boundary queued behind the exchange on the high-priority comm stream, split by sites") + "): span per apply")
        else:                   # one ghost-aware launch after the exchange
            kern_ms, n_launch = max_over_ranks(t_all / max(1, n_all)), n_all
            kname = f"{kstem}<lanes={lanes_n}, ghost=true> (all sites, after the exchange)"
        dom_sites = vh
        breakdown = {"pass": f"{nb} steps with per-kernel CUDA events after the timed region",
                     "interior_us": round(t_int / n_int * 1e3, 2) if n_int else None,
                     "boundary_us": round(t_bnd / n_bnd * 1e3, 2) if n_bnd else None,
                     "span_us": round(t_span / n_span * 1e3, 2) if n_span else None,
                     "exchange_us": round(t_x / n_x * 1e3, 2) if n_x else None,
                     "interior_sites": int(plan.interior_sites), "boundary_sites": int(plan.boundary_sites),
                     "launches_per_step": launches_per_step}
    achieved = algo_bytes_site * dom_sites / (kern_ms * 1e-3) / 1e9
    variant = (args.kernel + ("-stage" if args.stage else "") + ("" if args.precision == "f64" else f"-{args.precision}")
               + ("" if args.recon == 18 else f"-r{args.recon}") + (f"-n{nrhs}" if nrhs > 1 else "")
               + ("-blocked" if args.layout == "blocked" else ""))
    roof = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
            "frac": round(achieved / peak, 4), "traffic": ncu_traffic(variant, extent), "kernel": kname,
            "bytes_per_launch": algo_bytes_site * dom_sites, "bytes_per_site": algo_bytes_site,
            "avg_launch_us": round(kern_ms * 1e3, 2), "launches": n_launch, "peak_source": peak_src,
            "frac_of_nominal_8TBs": round(achieved / NOMINAL_HBM_GBS, 4)}
    if breakdown:
        roof["breakdown"] = breakdown

    # ---- end to end through the C ABI from pinned host buffers: every step copies its psi
    # host->device and its chi device->host (dslash_apply_host_batch pipelines the copies of
    # neighbouring steps against the compute on 3 device slots)
    e2e = None
    if not args.no_e2e and nrhs == 1:
        RH = 4
        hins = [torch.from_numpy(fieldgen.vector_cb(gdims, fieldgen.SEED_PSI + r, 1 - parity, origin=origin,
                                                    extent=extent)).to(D.dtype).pin_memory() for r in range(RH)]
        houts = [torch.empty_like(hins[0]).pin_memory() for _ in range(RH)]
        ke = max(12, min(args.steps, 600))
        seq_in = [hins[i % RH] for i in range(ke)]
        seq_out = [houts[i % RH] for i in range(ke)]
        D.apply_host_batch(seq_out[:6], seq_in[:6], parity, stream)       # warm-up (allocates slots)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        ev0.record(stream)
        D.apply_host_batch(seq_out, seq_in, parity, stream)
        ev1.record(stream)
        torch.cuda.synchronize()
        te = max_over_ranks(ev0.elapsed_time(ev1))
        e2e = {"value": round(FLOP_PER_SITE * total_sites * ke / (te * 1e-3) / 1e9, 2),
               "unit": "GFLOP/s", "h2d_bytes_per_step": vec_bytes * world, "d2h_bytes_per_step": vec_bytes * world,
               "steps": ke, "ms_per_step": te / ke,
               "path": "dslash_apply_host_batch (C ABI): per step pinned host psi -> device, apply, "
                       "device -> pinned host chi; copies of neighbouring steps overlap the compute"}

    # calibration in the same run: the achievable HBM READ bandwidth of this GPU now,
    # a plain reduction over a 2 GiB fp64 tensor (torch's kernel: a calibration, not the product),
    # after the timed region; the stencil streams 98% reads, so this is its tighter ceiling
    if not args.no_read_calibration:
        try:
            cal = torch.empty(2 ** 28, dtype=torch.float64, device="cuda").fill_(1.0)
            for _ in range(3):
                cal.sum()
            torch.cuda.synchronize()
            ca, cb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            ca.record()
            for _ in range(10):
                cal.sum()
            cb.record()
            torch.cuda.synchronize()
            rgbs = cal.numel() * 8 * 10 / (ca.elapsed_time(cb) * 1e-3) / 1e9
            roof["read_stream_gbs_same_run"] = round(rgbs, 1)
            roof["frac_of_read_stream"] = round(roof["achieved"] / rgbs, 4)
            del cal
        except Exception as exc:  # pragma: no cover - calibration is optional
            roof["read_stream_gbs_same_run"] = f"unavailable: {exc}"

    # ---- CPU oracle (rank 0; the product's result never depends on it).  N = 1: the 32^4 workload;
    # strong scaling: the global lattice (48^4); plus the 48^4 leg of SURVEY §8(d) unless skipped.
    cpu = None
    if rank == 0 and not args.no_cpu_baseline and (world == 1 or args.global_dims):
        cpu, _ = run_oracle_baseline(gdims, parity, args.cpu_seconds)
        if not args.no_oracle_48 and tuple(gdims) != (48, 48, 48, 48):
            cpu["legs"] = [oracle_leg((48, 48, 48, 48), parity, min(args.cpu_seconds, 8.0))]
    if world > 1:
        dist.barrier()

    if rank == 0:
        line = {"metric": METRIC, "value": round(gflops, 2), "unit": "GFLOP/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_max / args.steps,
                "higher_is_better": True, "scaling": "strong" if args.global_dims else "weak", "vs_baseline": None,
                "dtype": {"f64": "f64", "f32": "f32", "mixed": "f32 links, f64 vectors/accumulation"}[args.precision],
                "data": "synthetic",
                "config": {"workload": name, "global_dims": list(gdims), "local_dims": list(extent),
                           "proc_grid": list(grid),
                           "grid_rule": None if not args.global_dims or args.grid else
                           "choose_grid: t alone while Lt/N >= 12, else max interior fraction, fewest face bytes, larger Pt",
                           "parallelism": (f"t{grid[3]}" if grid[2] == 1 else f"z{grid[2]}t{grid[3]}")
                           + (f" self-halo mask {args.force_halo}" if args.force_halo else "")
                           + (" via NCCL send/recv to self" if args.force_halo and args.self_nccl else ""),
                           "parity": parity,
                           "kernel": args.kernel, "stage": bool(args.stage), "block": args.block or None,
                           "precision": args.precision, "long_link_recon": args.recon, "nrhs": nrhs,
                           "vector_layout": args.layout,
                           "overlap": "none" if args.no_overlap else args.overlap, "pdl": not args.no_pdl,
                           "halo_dryrun_results_invalid": True if args.halo_dryrun else None,
                           "per_kernel_events_in_timed_region": bool(args.flush_l2),
                           "transport": args.transport if world > 1 else None,
                           "colocated_ranks_on_one_gpu": bool(args.colocate) or None,
                           "l2": ("L2 flushed between steps (2x L2 buffer write); time = summed kernel events; "
                                  if args.flush_l2 else "") + f"inputs > L2: {(algo_bytes_site - 2 * vec_bytes // (3 * vh) * 3) * vh / 1e9:.2f} GB "
                                 f"links/apply streamed; {R} rotating (psi, chi) pairs = "
                                 f"{R * 2 * vec_bytes / 1e6:.0f} MB > {l2_bytes / 1e6:.0f} MB L2",
                           "links": "random SU(3) fat (seed 1), -1/24 random SU(3) long (seed 2)"},
                "algorithmic_gbs": round(algo_gbs, 1),
                "pct_hbm_measured": round(100 * algo_gbs / peak, 2),
                "pct_hbm_nominal_8TBs": round(100 * algo_gbs / NOMINAL_HBM_GBS, 2),
                "roofline": roof, "clocks": clk.summary(), "e2e": e2e,
                "gpu_launches": launches_per_step * args.steps,
                "cpu_baseline": cpu}
        sys.stdout.flush()
        os.dup2(real_stdout, 1)
        print(json.dumps(line), flush=True)
        os.dup2(2, 1)
    D.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
