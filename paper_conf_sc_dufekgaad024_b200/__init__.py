"""B200-native single-parity HISQ Dslash (MILC-Dslash hot path, Dufek et al. SC'24 workshops).

The product is the C-ABI library ``libhisq_dslash.so`` (include/hisq_dslash.h):
hand-written sm_100a CUDA kernels plus a C++ host runtime with an NCCL depth-3 halo
exchange.  This package is a thin Python binding: ``_abi`` exposes the C functions
under their own names (argument marshalling only) and :class:`Dslash` wraps a handle,
taking device memory and streams from PyTorch.  There is no CPU fallback: importing
without the built library raises.
"""
from __future__ import annotations

from . import _abi
from ._abi import (DSLASH_BOTH, DSLASH_EVEN, DSLASH_F64, DSLASH_KERNEL_DIR4, DSLASH_KERNEL_SITE,  # noqa: F401
                   DSLASH_ODD, DSLASH_OPT_BLOCK, DSLASH_OPT_FORCE_HALO, DSLASH_OPT_KERNEL, DSLASH_OPT_OVERLAP,
                   DSLASH_OPT_TIMING, DSLASH_TIMING_ALL, DSLASH_TIMING_BOUNDARY, DSLASH_TIMING_INTERIOR,
                   KERNELS, DslashError, dslash_plan)

FLOP_PER_SITE = 1146          # 600.8 MFLOP per 32^4 apply = 1146 per target site
LINK_BYTES_PER_SITE = 2304    # 16 matrices x 9 complex x 16 B (fp64), streamed once
ALGO_BYTES_PER_SITE = 2400    # + 48 B source (ideal reuse) + 48 B output
# algorithmic bytes per target site by precision: links + source + output
ALGO_BYTES = {"f64": 2304 + 48 + 48, "f32": 1152 + 24 + 24, "mixed": 1152 + 48 + 48}


def algo_bytes(precision="f64", recon=18, nrhs=1):
    """Algorithmic bytes per target site for one launch over nrhs right-hand sides: links
    (recon-12 stores 6 of 9 entries of the 8 long matrices, recon-9 4 + a shared phase entry) + nrhs x (source with ideal reuse +
    output)."""
    lb = 16 if precision == "f64" else 8
    vb = 8 if precision == "f32" else 16
    # recon-9: 4 entries per long matrix + the (psi_f, psi_b) pair per direction (one complex
    # entry in fp64, a whole float4 = two complex entries in the fp32 paired layout)
    r9 = 8 * 4 + (4 if precision == "f64" else 8)
    link_entries = 8 * 9 + (8 * 6 if recon == 12 else r9 if recon == 9 else 8 * 9)
    return link_entries * lb + nrhs * 2 * 3 * vb

__all__ = ["Dslash", "DslashError", "dslash_plan", "FLOP_PER_SITE", "ALGO_BYTES_PER_SITE"]


def _stream_handle(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)


class Dslash:
    """One handle of the library on the current CUDA device.

    precision: "f64" (default), "f32" (complex64 vectors and fp32 links) or "mixed"
    (fp32 links, complex128 vectors, fp64 accumulation).
    Vectors are torch complex128 (complex64 for "f32") CUDA tensors of shape (3, Vh_local) (colour-major,
    checkerboard site order cb = local lex // 2); links are canonical forward links
    (Lt, Lz, Ly, Lx, 4, 3, 3) complex128 over the local volume, numpy (host) or torch
    (device).  With ``world_size > 1`` the NCCL unique id is broadcast through the
    default torch.distributed process group.
    """

    def __init__(self, global_dims, proc_grid=(1, 1, 1, 1), parity_mask=DSLASH_BOTH, kernel="dir2", block=0,
                 force_halo=0, overlap=True, timing=False, rank=0, world_size=1, min_blocks=0, precision="f64",
                 recon=18, transport="nccl", pdl=True, self_nccl=False, stage=False, push=False):
        import torch
        self.global_dims = tuple(int(d) for d in global_dims)
        self.precision = precision
        self.dtype = torch.complex64 if precision == "f32" else torch.complex128
        self.proc_grid = tuple(int(p) for p in proc_grid)
        uid = None
        self.world_size, self.rank, self.transport = world_size, rank, transport
        # an NCCL communicator for the halo (transport "nccl") and, on an NCCL process group, for
        # the solver's cross-rank dot products even when the halo goes through P2P
        use_nccl = False
        if world_size > 1:
            import torch.distributed as dist
            use_nccl = transport == "nccl" or dist.get_backend() == "nccl"
        if use_nccl:
            import torch
            import torch.distributed as dist
            t = torch.zeros(128, dtype=torch.uint8, device="cuda" if dist.get_backend() == "nccl" else "cpu")
            if rank == 0:
                t.copy_(torch.frombuffer(bytearray(_abi.dslash_get_unique_id()), dtype=torch.uint8))
            dist.broadcast(t, 0)
            uid = bytes(t.cpu().numpy().tobytes())
        elif self_nccl:
            # one rank: a one-rank communicator, and the self-neighbour faces go through NCCL
            # send/recv to this rank (the P = 2 message pattern on one GPU)
            assert world_size == 1 and transport == "nccl", "self_nccl is a one-rank NCCL-transport option"
            uid = _abi.dslash_get_unique_id()
        # the library links its own CUDA runtime: bind the handle to torch's current device explicitly
        _abi.dslash_set_device(torch.cuda.current_device())
        self.h = _abi.dslash_create(self.global_dims, self.proc_grid, parity_mask, _abi.PRECISIONS[precision], uid,
                                    world_size, rank)
        try:
            _abi.dslash_set_option(self.h, DSLASH_OPT_KERNEL, KERNELS[kernel] if isinstance(kernel, str) else kernel)
            if block:
                _abi.dslash_set_option(self.h, DSLASH_OPT_BLOCK, block)
            if min_blocks:
                _abi.dslash_set_option(self.h, _abi.DSLASH_OPT_MIN_BLOCKS, min_blocks)
            if recon != 18:
                _abi.dslash_set_option(self.h, _abi.DSLASH_OPT_LONG_RECON, recon)
            _abi.dslash_set_option(self.h, _abi.DSLASH_OPT_PDL, int(bool(pdl)))
            if transport == "p2p" and (world_size == 1 or use_nccl):
                _abi.dslash_set_option(self.h, _abi.DSLASH_OPT_TRANSPORT, _abi.DSLASH_TRANSPORT_P2P)
            if push:  # producer push: two ghost banks, allocated before they are IPC-exported
                _abi.dslash_set_option(self.h, _abi.DSLASH_OPT_PUSH, 1)
            if transport == "p2p":
                if world_size > 1:      # exchange CUDA IPC handles through torch.distributed
                    import torch.distributed as dist
                    blobs = [None] * world_size
                    dist.all_gather_object(blobs, _abi.dslash_get_ipc_blob(self.h))
                    _abi.dslash_open_ipc_blobs(self.h, b"".join(blobs))
            if force_halo:
                _abi.dslash_set_option(self.h, DSLASH_OPT_FORCE_HALO, force_halo)
            if self_nccl:
                _abi.dslash_set_option(self.h, _abi.DSLASH_OPT_SELF_NCCL, 1)
            if stage:
                _abi.dslash_set_option(self.h, _abi.DSLASH_OPT_STAGE, 1)
            # True / "sites": split by sites (default); "dirs": split by direction; False / "none"
            _abi.dslash_set_option(self.h, DSLASH_OPT_OVERLAP,
                                   _abi.OVERLAPS[overlap] if isinstance(overlap, str) else int(overlap))
            if timing:
                _abi.dslash_set_option(self.h, DSLASH_OPT_TIMING, 1)
        except Exception:
            self.close()
            raise
        self.plan = _abi.dslash_get_plan(self.h)
        self.vh = int(self.plan.vh_local)
        self.local_dims = tuple(self.plan.local_dims)
        self.origin = tuple(self.plan.origin)

    # -- links
    def load_links(self, fat, lng, stream=None):
        import numpy as np
        if isinstance(fat, np.ndarray):
            fat = np.ascontiguousarray(fat, dtype=np.complex128)
            lng = np.ascontiguousarray(lng, dtype=np.complex128)
            self._check_links(fat.shape, lng.shape)
            _abi.dslash_load_links(self.h, fat.ctypes.data, lng.ctypes.data, 0, _stream_handle(stream))
        else:
            import torch
            assert fat.is_cuda and fat.dtype == torch.complex128 and fat.is_contiguous()
            assert lng.is_cuda and lng.dtype == torch.complex128 and lng.is_contiguous()
            self._check_links(tuple(fat.shape), tuple(lng.shape))
            _abi.dslash_load_links(self.h, fat.data_ptr(), lng.data_ptr(), 1, _stream_handle(stream))

    def get_links(self, parity):
        """Internal link arrays of target parity as numpy (Vh, 4 mu, 4 l, 3, 3) complex128,
        l = F(x,mu), F(x-mu,mu)^dag, N(x,mu), N(x-3mu,mu)^dag (verification of load_links)."""
        import numpy as np
        out = np.empty((self.vh, 4, 4, 3, 3), np.complex128)
        _abi.dslash_get_links(self.h, int(parity), out.ctypes.data)
        return out

    def _check_links(self, a, b):
        lx, ly, lz, lt = self.local_dims
        want = (lt, lz, ly, lx, 4, 3, 3)
        if tuple(a) != want or tuple(b) != want:
            raise ValueError(f"links must have shape {want}, got {a} and {b}")

    # -- vectors
    def empty_vector(self):
        import torch
        return torch.empty((3, self.vh), dtype=self.dtype, device="cuda")

    def _check_vec(self, v, cuda=True):
        if not (v.is_cuda == cuda and v.dtype == self.dtype and v.is_contiguous() and tuple(v.shape) == (3, self.vh)):
            where = "CUDA" if cuda else "CPU"
            raise ValueError(f"vector must be a contiguous {self.dtype} {where} tensor of shape (3, {self.vh})")

    def apply(self, out, inp, parity, stream=None):
        """out = D inp on target parity `parity` (stream-ordered, asynchronous)."""
        self._check_vec(out)
        self._check_vec(inp)
        _abi.dslash_apply(self.h, out.data_ptr(), inp.data_ptr(), int(parity), _stream_handle(stream))
        return out

    def apply_push(self, out, inp, parity, stream=None):
        """out = D inp, and the faces of out go straight into the neighbours' ghosts (push=True):
        the next apply on every rank must take ``out`` as its source."""
        self._check_vec(out)
        self._check_vec(inp)
        _abi.dslash_apply_push(self.h, out.data_ptr(), inp.data_ptr(), int(parity), _stream_handle(stream))
        return out

    def apply_multi(self, out, inp, parity, stream=None):
        """out[r] = D inp[r] for tensors of shape (nrhs, 3, Vh), one pass over the links."""
        for v in (out, inp):
            if not (v.is_cuda and v.dtype == self.dtype and v.is_contiguous() and v.dim() == 3
                    and tuple(v.shape[1:]) == (3, self.vh)):
                raise ValueError(f"multi-RHS vectors must be contiguous {self.dtype} CUDA tensors (n, 3, {self.vh})")
        if out.shape[0] != inp.shape[0]:
            raise ValueError("out and inp hold different numbers of right-hand sides")
        _abi.dslash_apply_multi(self.h, int(inp.shape[0]), out.data_ptr(), inp.data_ptr(), int(parity),
                                _stream_handle(stream))
        return out

    def _check_blocked(self, *vs):
        n = vs[0].numel()
        for v in vs:
            if not (v.is_cuda and v.dtype == self.dtype and v.is_contiguous() and v.numel() == n
                    and n % (3 * self.vh) == 0):
                raise ValueError(f"site-blocked vectors must be contiguous {self.dtype} CUDA tensors of "
                                 f"nrhs x 3 x {self.vh} elements")
        return n // (3 * self.vh)

    def apply_multi_blocked(self, out, inp, parity, stream=None):
        """out = D inp for nrhs right-hand sides in the site-blocked layout (dslash_apply_multi_blocked:
        element (r, c, cb) at [cb // 16][r * 3 + c][cb % 16]); tensors of nrhs x 3 x Vh elements."""
        nrhs = self._check_blocked(out, inp)
        _abi.dslash_apply_multi_blocked(self.h, nrhs, out.data_ptr(), inp.data_ptr(), int(parity),
                                        _stream_handle(stream))
        return out

    def to_blocked(self, blocked, planar, stream=None):
        """planar (nrhs, 3, Vh) -> site-blocked copy (on the device, stream-ordered)."""
        nrhs = self._check_blocked(blocked, planar)
        _abi.dslash_vectors_to_blocked(self.h, nrhs, blocked.data_ptr(), planar.data_ptr(), _stream_handle(stream))
        return blocked

    def from_blocked(self, planar, blocked, stream=None):
        """site-blocked -> planar (nrhs, 3, Vh) copy (on the device, stream-ordered)."""
        nrhs = self._check_blocked(planar, blocked)
        _abi.dslash_vectors_from_blocked(self.h, nrhs, planar.data_ptr(), blocked.data_ptr(), _stream_handle(stream))
        return planar

    def normal_apply(self, out, inp, parity, mass, stream=None):
        """out = (m^2 - D_{p,1-p} D_{1-p,p}) inp on parity p (needs parity_mask BOTH, fp64 vectors)."""
        self._check_vec(out)
        self._check_vec(inp)
        _abi.dslash_normal_apply(self.h, out.data_ptr(), inp.data_ptr(), int(parity), float(mass),
                                 _stream_handle(stream))
        return out

    def cg(self, x, b, parity, mass, rel_tol=1e-10, max_iter=1000, stream=None):
        """Solve (m^2 - D_{p,1-p} D_{1-p,p}) x = b by CG; returns (converged, iterations, true rel. residual)."""
        self._check_vec(x)
        self._check_vec(b)
        st, it, res = _abi.dslash_cg(self.h, x.data_ptr(), b.data_ptr(), int(parity), float(mass), float(rel_tol),
                                     int(max_iter), _stream_handle(stream))
        return st == _abi.DSLASH_OK, it, res

    def cg_multi_blocked(self, x, b, parity, mass, rel_tol=1e-10, max_iter=1000, stream=None):
        """CG for nrhs <= 8 systems sharing every link pass (dslash_cg_multi_blocked); x, b: site-blocked
        fp64 tensors of nrhs x 3 x Vh elements.  Returns (all converged, [iterations], [true rel. residual])."""
        nrhs = self._check_blocked(x, b)
        st, its, res = _abi.dslash_cg_multi_blocked(self.h, nrhs, x.data_ptr(), b.data_ptr(), int(parity), float(mass),
                                                    float(rel_tol), int(max_iter), _stream_handle(stream))
        return st == _abi.DSLASH_OK, its, res

    def cg_mixed(self, x, b, parity, mass, rel_tol=1e-10, inner_tol=1e-4, max_iter=5000, stream=None):
        """Mixed-precision CG (fp32 inner solves, fp64 defect correction) for the same system as
        cg(); returns (converged, inner iterations, outer corrections, true rel. residual)."""
        self._check_vec(x)
        self._check_vec(b)
        st, it, outer, res = _abi.dslash_cg_mixed(self.h, x.data_ptr(), b.data_ptr(), int(parity), float(mass),
                                                  float(rel_tol), float(inner_tol), int(max_iter),
                                                  _stream_handle(stream))
        return st == _abi.DSLASH_OK, it, outer, res

    def __call__(self, inp, parity, stream=None):
        return self.apply(self.empty_vector(), inp, parity, stream)

    def apply_host(self, out, inp, parity, stream=None):
        """Host-buffer path (end-to-end): torch CPU complex128 tensors (pin them for async copies)."""
        for v in (out, inp):
            self._check_vec(v, cuda=False)
        _abi.dslash_apply_host(self.h, out.data_ptr(), inp.data_ptr(), int(parity), _stream_handle(stream))
        return out

    def apply_host_batch(self, outs, inps, parity, stream=None):
        """Pipelined host-buffer applies: outs[i] = D inps[i] (torch CPU complex128, pinned)."""
        for v in list(outs) + list(inps):
            self._check_vec(v, cuda=False)
        _abi.dslash_apply_host_batch(self.h, [o.data_ptr() for o in outs], [v.data_ptr() for v in inps],
                                     int(parity), _stream_handle(stream))
        return outs

    def kernel_timing(self, which=DSLASH_TIMING_ALL):
        """(total ms, launches) of the kernels of class `which` recorded since the last reset."""
        return _abi.dslash_kernel_timing(self.h, which)

    def timeline(self, max_entries=4096):
        """Recorded intervals in record order: [(kind name, start_ms, end_ms)] relative to the
        first one since the last reset (timing=True): kernels, spans and halo exchanges."""
        return [(_abi.TIMING_KINDS.get(k, k), a, b) for k, a, b in _abi.dslash_timeline(self.h, max_entries)]

    def kernel_timing_reset(self):
        _abi.dslash_kernel_timing_reset(self.h)

    def sync(self):
        _abi.dslash_sync(self.h)

    def close(self):
        if getattr(self, "h", None):
            _abi.dslash_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()
