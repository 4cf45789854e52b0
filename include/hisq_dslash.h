/*
 * hisq_dslash.h -- C ABI of the B200-native single-parity HISQ (improved-staggered)
 * Dslash library (libhisq_dslash.so, sm_100a).
 *
 * The operation (§II, Eq. (1) "C = Dslash x B", with the third-
 * neighbour Naik terms of L27/L51; readings Z1-Z10): for every local
 * site x of the target parity p,
 *
 *   chi(x) = sum_{mu=0..3} [  F(x,mu) psi(x+mu)   - F(x-mu,mu)^dag  psi(x-mu)
 *                           + N(x,mu) psi(x+3mu)  - N(x-3mu,mu)^dag psi(x-3mu) ]
 *
 * on a periodic 4-D lattice, fp64 complex.  F = fat links, N = long (Naik) links,
 * psi lives on parity 1-p (target sites s* in [0, L^4/2)).
 *
 * Conventions (all functions):
 *   - dims are {Lx, Ly, Lz, Lt}, x fastest; lex(x,y,z,t) = x + Lx*(y + Ly*(z + Lz*t));
 *     parity p(x) = (x+y+z+t) mod 2 in GLOBAL coordinates.
 *   - Complex numbers are two interleaved reals (re, im): 16 B (fp64), or 8 B for the
 *     vectors of a DSLASH_F32 handle.
 *   - Vector layout (in, out): [3][Vh_local] complex, colour-major ("SoA"), where the
 *     checkerboard index cb = (local lex) / 2 enumerates the local sites of one parity
 *     in lexicographic order (Z8).  Vh_local = local volume / 2.
 *   - Canonical link layout (load_links input): [t][z][y][x][mu][3][3] complex over the
 *     LOCAL volume, forward links only, row-major 3x3 (|i| x |j| complex
 *     matrices, an array of L^4 x |k| per link kind).
 *   - Every function returns a dslash_status; no C++ exception crosses the ABI.  Errors
 *     are sticky per handle: once a call fails, dslash_error_string(h) describes the
 *     first failure; later calls still run their own argument checks.
 *   - Streams are cudaStream_t passed as void* (NULL = the legacy default stream).
 *
 * Multi-GPU: one process per GPU; the lattice may be split along
 * z and t only (proc_grid = {1, 1, Pz, Pt}); rank = cz + Pz * ct.  Each apply exchanges
 * a depth-3 halo of the source parity (the Naik hop reaches 3 sites) with NCCL
 * send/recv on an internal communication stream, overlapped with the interior kernel.
 */
#ifndef HISQ_DSLASH_H
#define HISQ_DSLASH_H

#include <stdint.h>

#if defined(__GNUC__)
#define DSLASH_API __attribute__((visibility("default")))
#else
#define DSLASH_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct dslash_s* dslash_t;
typedef void* dslash_stream_t; /* cudaStream_t */

typedef enum {
    DSLASH_OK = 0,
    DSLASH_ERR_ARG = 1,         /* invalid argument (odd/small extents, bad parity, NULL/aliased pointers) */
    DSLASH_ERR_STATE = 2,       /* call out of order (apply before load_links, option after load_links) */
    DSLASH_ERR_CUDA = 3,        /* a CUDA runtime call failed (message carries cudaGetErrorString) */
    DSLASH_ERR_NCCL = 4,        /* an NCCL call failed */
    DSLASH_ERR_OOM = 5,         /* device allocation failed */
    DSLASH_ERR_UNSUPPORTED = 6, /* valid but not implemented (x/y partitioning, an fp32 solver) */
    DSLASH_ERR_NOT_CONVERGED = 7 /* dslash_cg reached max_iter (not sticky; results are still written) */
} dslash_status;

enum { DSLASH_EVEN = 0, DSLASH_ODD = 1, DSLASH_BOTH = 2 }; /* parity_mask */
/* precision: F64 = fp64 links, vectors and arithmetic (the paper's, L278); F32 = fp32 links
 * and vectors (complex64), fp32 accumulation; MIXED = fp32 links, fp64 vectors and fp64
 * accumulation (links are widened before the FMAs).  load_links always takes fp64 input. */
enum { DSLASH_F64 = 0, DSLASH_F32 = 1, DSLASH_MIXED = 2 };

/* Kernel variants (DSLASH_OPT_KERNEL); DESIGN.md §Kernels. */
enum {
    DSLASH_KERNEL_SITE = 0, /* one thread per target site, 16 link matrices streamed per thread   */
    DSLASH_KERNEL_DIR4 = 1, /* four lanes per site (one per mu), 2-step shuffle reduction ("3LP") */
    DSLASH_KERNEL_DIR2 = 2  /* two lanes per site (two directions each), 1-step shuffle reduction  */
};

/* Options (dslash_set_option). */
enum {
    DSLASH_OPT_KERNEL = 0,      /* kernel variant (default DSLASH_KERNEL_DIR2); before load_links, as
                                   it fixes the link layout                                            */
    DSLASH_OPT_BLOCK = 1,       /* threads per block (multiple of 32, <= 256), 0 = default; any time   */
    DSLASH_OPT_FORCE_HALO = 2,  /* bitmask of directions (bit mu) exchanged through the halo path even
                                   when Pmu == 1 (self-halo: neighbour = self); before load_links      */
    DSLASH_OPT_OVERLAP = 3,     /* how an apply with a halo overlaps the exchange (DSLASH_OVERLAP_*);
                                   any time                                                           */
    DSLASH_OPT_TIMING = 4,      /* 1: record CUDA events around every kernel (dslash_kernel_timing)   */
    DSLASH_OPT_LONG_RECON = 6,  /* 18 (default): long links stored in full; 12: long links stored as
                                   rows 0 and 1 only, row 2 rebuilt in registers as conj(r0 x r1)/s
                                   (QUDA "recon-12").  Requires every long link
                                   (and the link halo) to be s*W with W in SU(3) and one real s;
                                   load_links verifies it and returns DSLASH_ERR_ARG otherwise.
                                   9: each long matrix M = s e^{i psi} W (W in SU(3), one real s
                                   per handle) stored as the 8 parameters of W (arg a1, arg c1, a2,
                                   a3, b1) + psi, rebuilt in registers (QUDA "recon-9"; accepts
                                   folded staggered signs and U(1) phases).  Register kernels, all
                                   precisions (dslash_cg_mixed's fp32 copies are rebuilt in full);
                                   load_links
                                   verifies that every long link
                                   is rebuilt within 1e-11 s, which also rejects links near the
                                   parameterisation's singular set |a2|^2 + |a3|^2 -> 0 (e.g.
                                   multiples of the identity): DSLASH_ERR_ARG.
                                   Before load_links                                                  */
    DSLASH_OPT_TRANSPORT = 8,   /* DSLASH_TRANSPORT_NCCL / _P2P; before load_links                    */
    DSLASH_OPT_PDL = 9,         /* 1 (default): launch the stencil kernels with programmatic stream
                                   serialization, so an apply's blocks start (and prefetch their
                                   first read-only link matrix) while the previous kernel on the
                                   stream drains; psi / chi are touched only after
                                   griddepcontrol.wait.  0: ordinary launches; any time              */
    DSLASH_OPT_SELF_NCCL = 10,  /* 1: directions whose neighbour is this rank (FORCE_HALO with Pmu == 1)
                                   exchange their faces (and load_links its link slabs) with NCCL
                                   send/recv to this rank instead of device copies: the message
                                   pattern of Pmu == 2, run on one GPU.  Needs the NCCL transport
                                   and a communicator (dslash_create with an id, also for
                                   nranks == 1); before load_links; 0 (default) = device copies    */
    DSLASH_OPT_STAGE = 11,      /* 1: neighbour-staged kernel for the site / dir2 variants (PAPER.md L321,
                                   the 3LP-1 local-memory staging): a block owns TY full x-rows of one
                                   (z, t); the TMA engine copies the source rows y0-3 .. y0+TY+2 into
                                   shared memory once (cp.async.bulk + mbarrier) and the 8 x/y hops
                                   per site read them there; z/t hops stay global loads.  Same link
                                   layout (any time).  An x-row must be a multiple of 16 bytes
                                   (fp32 vectors: Lx/2 even), else DSLASH_ERR_UNSUPPORTED, also at
                                   apply time when dslash_cg_mixed runs the handle in fp32.
                                   0 (default): off                                                 */
    DSLASH_OPT_HALO_DRYRUN = 13,/* timing aid (NCCL / device-copy transport): halo_start keeps its
                                   events and stream order but moves no bytes, so the ghost faces
                                   are stale and results WRONG; prices an overlap scheme without the
                                   exchange itself; any time                                        */
    DSLASH_OPT_PUSH = 14,       /* 1: producer push (P2P transport only; before load_links and the IPC
                                   setup).  The ghosts get two banks (epoch e reads bank e & 1) and
                                   dslash_apply_push / the normal operator / CG store the depth-3
                                   faces of an apply's OUTPUT straight into the neighbours' ghosts
                                   from the stencil kernel's epilogue (peer memory over NVLink), so
                                   the next apply, whose source that output is, moves no bytes.
                                   0 (default): off                                                 */
    DSLASH_OPT_MIN_BLOCKS = 5   /* register budget of the stencil kernel, as the minimum number of
                                   resident 256-thread blocks per SM: 2 (<= 128 registers), 3 (<= 80),
                                   4 (<= 64); 0 = default; any time                                    */
};

/* Overlap modes (DSLASH_OPT_OVERLAP) of an apply that exchanges a halo. */
enum {
    DSLASH_OVERLAP_NONE = 0,   /* one kernel over all sites after the exchange                        */
    DSLASH_OVERLAP_SITES = 1,  /* (default) split by sites: the interior box (no ghost source) runs
                                  during the exchange; the boundary slabs run on a high-priority
                                  stream once the faces land                                        */
    DSLASH_OVERLAP_DIRS = 2    /* split by direction: a local pass over every site during the
                                  exchange skips the hops into ghost faces; a ghost pass over the
                                  boundary slabs then adds exactly those hops to the stored partial
                                  sums (+96 B per boundary site).  Hides the exchange even when no
                                  site is interior (local extent 6 with a depth-3 halo).  Boundary
                                  sites sum their terms in another order than DSLASH_OVERLAP_NONE:
                                  equal within the fp64 tolerance, not bitwise                      */
};

/* Halo transports (DSLASH_OPT_TRANSPORT). */
enum {
    DSLASH_TRANSPORT_NCCL = 0, /* grouped ncclSend/ncclRecv on the communication stream (default when
                                  dslash_create got an NCCL unique id)                               */
    DSLASH_TRANSPORT_P2P = 1   /* SM-free: faces are copied by the copy engines straight into the
                                  neighbours' CUDA-IPC-mapped ghost buffers (NVLink within a node),
                                  and cuStreamWriteValue32/WaitValue32 epoch flags order producers and
                                  consumers.  Needs dslash_get_ipc_blob / dslash_open_ipc_blobs before
                                  load_links when neighbours are other ranks; load_links then copies
                                  its top link slices into the plus neighbours' IPC-mapped slab
                                  buffers itself, and the solver's dot products are summed through
                                  the ranks' IPC-mapped control blocks.  Also works for several ranks
                                  on ONE GPU (NCCL refuses that).  At most 8 right-hand sides per
                                  apply                                                              */
};

/* Kernel classes for dslash_kernel_timing.  SPAN: with a halo and the classic split, the time
 * from the interior kernel's start to the join after the (overlapping, higher-priority) boundary
 * kernel, i.e. the duration of the apply's stencil work; EXCHANGE: the halo exchange on the
 * communication stream (NCCL send/recv, device copies or P2P copies, from the comm stream's
 * start of the exchange to its end); ALL sums the kernel launches only. */
enum { DSLASH_TIMING_INTERIOR = 0, DSLASH_TIMING_BOUNDARY = 1, DSLASH_TIMING_ALL = 2, DSLASH_TIMING_SPAN = 3,
       DSLASH_TIMING_EXCHANGE = 4 };

/* Host-only decomposition of the local lattice (no CUDA calls).  A "box" is
 * [lo[d], hi[d]) per dimension in local coordinates; the target-parity sites of a
 * box number (hi0-lo0)/2 * (hi1-lo1) * (hi2-lo2) * (hi3-lo3). */
typedef struct {
    int32_t lo[4];
    int32_t hi[4];
} dslash_box_t;

typedef struct {
    int32_t global_dims[4];
    int32_t proc_grid[4];
    int32_t proc_coords[4];
    int32_t local_dims[4];
    int32_t origin[4];         /* global coordinate of local (0,0,0,0); always even */
    int32_t halo[4];           /* 1 if direction mu exchanges a depth-3 halo        */
    int32_t nbr_rank[4][2];    /* [mu][0 = minus, 1 = plus] neighbour rank (self if Pmu == 1) */
    int32_t rank, nranks;
    int64_t vh_local;          /* local target (= source) sites per parity           */
    int64_t face_vh[4];        /* source sites in one depth-3 face slab (0 if no halo) */
    int32_t n_interior, n_boundary;
    dslash_box_t interior[1];  /* sites whose 16 sources are all local               */
    dslash_box_t boundary[4];  /* the remaining sites (disjoint boxes)               */
    int64_t interior_sites, boundary_sites;
} dslash_plan_t;

/* Compute the decomposition for `rank` of `nranks` (no CUDA, no allocation).
 * force_halo_mask: as DSLASH_OPT_FORCE_HALO.  Errors: DSLASH_ERR_ARG for odd or < 2
 * extents, a halo direction with an odd local extent or one < 4 (depth-3 halo plus
 * parity), extents not divisible by proc_grid, prod(proc_grid) != nranks, rank out of
 * range; DSLASH_ERR_UNSUPPORTED for proc_grid[0] or proc_grid[1] != 1. */
DSLASH_API dslash_status dslash_plan(const int32_t global_dims[4], const int32_t proc_grid[4], int32_t rank,
                          int32_t nranks, int32_t force_halo_mask, dslash_plan_t* plan);

/* Create a handle on the current CUDA device.  parity_mask selects for which target
 * parities links are prepared (DSLASH_BOTH doubles link memory).  precision: DSLASH_F64,
 * DSLASH_F32 or DSLASH_MIXED (it fixes the stored link type and the vector type).
 * nccl_unique_id: the 128-byte ncclUniqueId from dslash_get_unique_id() on rank 0,
 * broadcast to all ranks by the caller; NULL when nranks == 1, or when the ranks will use
 * DSLASH_TRANSPORT_P2P (then no NCCL communicator is created).  With nranks == 1 an id
 * creates a one-rank communicator (for DSLASH_OPT_SELF_NCCL; the solver's sums then also
 * pass through ncclAllReduce).  On success *out owns
 * a CUDA communication stream, events, ghost buffers and (nranks > 1) an NCCL
 * communicator; release it with dslash_destroy.  On failure *out is NULL. */
DSLASH_API dslash_status dslash_create(const int32_t global_dims[4], const int32_t proc_grid[4], int32_t parity_mask,
                            int32_t precision, const void* nccl_unique_id, int32_t nranks, int32_t rank,
                            dslash_t* out);

/* P2P transport setup.  dslash_ipc_blob_size() bytes describe one rank's buffers (CUDA IPC
 * handles of its ghost buffers, its link-slab receive buffers and its control block of epoch
 * flags and reduction slots; the library allocates them, library-owned like the ghosts).  Every
 * rank writes its blob with dslash_get_ipc_blob, the caller all-gathers them (blobs of rank r at
 * r * size) and every rank calls dslash_open_ipc_blobs once, which maps every rank's control
 * block and the neighbours' buffers.  Both need DSLASH_OPT_TRANSPORT = P2P (and DSLASH_OPT_PUSH,
 * if wanted) first.  Ranks must be on GPUs of one node (or the same GPU).  Errors:
 * DSLASH_ERR_ARG for a malformed or misordered blob (e.g. from another library version),
 * DSLASH_ERR_STATE for a second dslash_open_ipc_blobs. */
DSLASH_API int64_t dslash_ipc_blob_size(void);
DSLASH_API dslash_status dslash_get_ipc_blob(dslash_t h, void* blob);
DSLASH_API dslash_status dslash_open_ipc_blobs(dslash_t h, const void* blobs);

/* Device selection for callers without their own CUDA runtime (e.g. plain C): the library
 * links its own copy of the CUDA runtime, so these act on the library's current device of the
 * calling thread, the device dslash_create binds a handle to.  dslash_set_device wraps
 * cudaSetDevice (DSLASH_ERR_ARG for an index out of range, DSLASH_ERR_CUDA otherwise);
 * dslash_device_count returns the number of visible devices (0 when none or on error).  Call
 * them before any other CUDA use in a forked child process. */
DSLASH_API dslash_status dslash_set_device(int32_t device);
DSLASH_API int32_t dslash_device_count(void);

/* Write a fresh ncclUniqueId (128 bytes) to id_out.  Call on rank 0 only. */
DSLASH_API dslash_status dslash_get_unique_id(void* id_out);

/* Set an option (see DSLASH_OPT_*).  DSLASH_ERR_STATE if the option must precede
 * load_links and links are loaded; DSLASH_ERR_ARG for unknown keys or bad values. */
DSLASH_API dslash_status dslash_set_option(dslash_t h, int32_t key, int64_t value);

/* Copy the caller's forward links into the library's internal parity-split layout,
 * building the back-links F(x-mu,mu)^dag and N(x-3mu,mu)^dag (|l| = 4
 * link arrays; Z2).  fat, lng: canonical layout over the local volume,
 * fp64 complex; on_device = 1 if they are device pointers, 0 for host memory.  When
 * partitioned, every rank sends its top 3 link slices of each halo direction to its plus
 * neighbour and receives the 3 slices below its origin from its minus neighbour: NCCL
 * send/recv, or, with DSLASH_TRANSPORT_P2P, copy-engine copies straight into the plus
 * neighbour's IPC-mapped slab buffer ordered by epoch flags (every rank of the partition must
 * call load_links; DSLASH_ERR_STATE if the IPC blobs were not opened).
 * Synchronous: on return the caller may free fat and lng.  Callable again to replace
 * the links (collectively). */
DSLASH_API dslash_status dslash_load_links(dslash_t h, const void* fat, const void* lng, int32_t on_device,
                                dslash_stream_t stream);

/* load_links with caller-provided link halo: for every halo direction d whose neighbour is
 * another rank, slab_fat[d] / slab_lng[d] hold the 3 coordinate slices just below the local
 * origin, taken from the minus neighbour's canonical links (its top 3 slices): layout
 * [d][z][y][x][mu][3][3] for d = t (3), [t][d][y][x][mu][3][3] for d = z (2).  Entries of other
 * directions are ignored (may be NULL).  Same device-ness as fat and lng (on_device).  For
 * callers that already hold the neighbours' slices (no exchange happens). */
DSLASH_API dslash_status dslash_load_links_halo(dslash_t h, const void* fat, const void* lng,
                                                const void* const slab_fat[4], const void* const slab_lng[4],
                                                int32_t on_device, dslash_stream_t stream);

/* Read back the internal link arrays of target parity `parity` (debugging / verification of
 * load_links): out_host[cb][mu][l][3][3] complex fp64, Vh_local x 144 complex, with
 * l = 0 F(x,mu), 1 F(x-mu,mu)^dag, 2 N(x,mu), 3 N(x-3mu,mu)^dag (PAPER.md L51's |l| = 4 arrays)
 * for the target site x of checkerboard index cb.  Values as stored (fp32 widened); with
 * recon-12 row 2 of the long matrices is not stored and reads as 0; with recon-9 the long
 * matrices are returned rebuilt from their stored parameters.  Synchronous. */
DSLASH_API dslash_status dslash_get_links(dslash_t h, int32_t parity, void* out_host);

/* chi = D psi on target parity `parity`.  out: device [3][Vh_local] complex on parity
 * `parity`; in: device [3][Vh_local] complex on parity 1-parity.  Both caller-owned,
 * 16-byte aligned, non-overlapping.  Stream-ordered and asynchronous: it runs
 * halo_start / interior kernel / halo_wait / boundary kernel internally.  Errors:
 * DSLASH_ERR_STATE before load_links, DSLASH_ERR_ARG for parity not in parity_mask,
 * NULL, misaligned or overlapping buffers. */
DSLASH_API dslash_status dslash_apply(dslash_t h, void* out, const void* in, int32_t parity, dslash_stream_t stream);

/* nrhs applies sharing one pass over the links: out and in hold nrhs
 * vectors back to back, [nrhs][3][Vh_local] (same element type and rules as dslash_apply),
 * out[r] = D in[r].  Every link is read from HBM once per launch of up to 8 right-hand
 * sides, so the algorithmic bytes per site are links + nrhs x (source + output).  The halo
 * exchange (N > 1) moves all nrhs faces at once. */
DSLASH_API dslash_status dslash_apply_multi(dslash_t h, int32_t nrhs, void* out, const void* in, int32_t parity,
                                            dslash_stream_t stream);

/* dslash_apply_multi on SITE-BLOCKED vectors (same operation, PAPER.md L45-51 for every right-hand
 * side; the L25 intensity argument for sharing the links): element (rhs r, colour c) of the
 * site with checkerboard index cb lies at
 *     [(cb / 16) * (nrhs * 3 * 16) + (r * 3 + c) * 16 + cb % 16]
 * (complex of the handle's vector precision), i.e. blocks of 16 consecutive sites, each holding
 * its nrhs x 3 rows of 16 back to back.  A warp's gathers of one hop then read a few contiguous
 * kilobytes instead of 3 x nrhs planes Vh_local apart, and one thread can hold all 8 right-hand
 * sides (8 RHS at 32^4: fp64 391 -> 355 us, fp32 219 -> 166 us; profiles/r03/blocked/).  Results
 * are bitwise those of dslash_apply_multi on the planar copies.  Caller-owned device buffers of nrhs x 3 x Vh_local complex, 16-byte aligned,
 * non-overlapping.  Requires Vh_local % 16 == 0.  With a halo (t and/or z partition, or a
 * forced self-halo) the faces are exchanged as whole blocks, in the same layout: every face must
 * be whole 16-site blocks (t: 3 Lx/2 Ly Lz; z: 3 Lx/2 Ly and Lx/2 Ly Lz multiples of 16, local
 * extents), and neither the producer push nor the split-by-direction overlap is available.
 * Otherwise DSLASH_ERR_UNSUPPORTED; other errors as dslash_apply_multi. */
DSLASH_API dslash_status dslash_apply_multi_blocked(dslash_t h, int32_t nrhs, void* out, const void* in,
                                                    int32_t parity, dslash_stream_t stream);

/* Layout conversion for dslash_apply_multi_blocked, stream-ordered on the device:
 * planar [nrhs][3][Vh_local] <-> site-blocked (above), complex of the handle's vector
 * precision.  Caller-owned, non-overlapping device buffers; Vh_local % 16 == 0, else
 * DSLASH_ERR_UNSUPPORTED. */
DSLASH_API dslash_status dslash_vectors_to_blocked(dslash_t h, int32_t nrhs, void* blocked, const void* planar,
                                                   dslash_stream_t stream);
DSLASH_API dslash_status dslash_vectors_from_blocked(dslash_t h, int32_t nrhs, void* planar, const void* blocked,
                                                     dslash_stream_t stream);

/* The same operation from HOST buffers (end-to-end path): copies in (host) to an
 * internal device buffer, applies, copies the result to out (host), all ordered on
 * `stream`; returns after enqueueing (synchronise the stream before reading out).
 * Pinned host memory gives asynchronous copies. */
DSLASH_API dslash_status dslash_apply_host(dslash_t h, void* out_host, const void* in_host, int32_t parity,
                                dslash_stream_t stream);

/* n applies from HOST buffers, pipelined: apply i reads in_host[i] and writes out_host[i]
 * (all [3][Vh_local] complex, pinned for overlap; inputs must not alias outputs).  The
 * host->device copy of apply i+1 and the device->host copy of apply i-1 run on internal
 * copy streams while apply i computes on `stream`, through 3 rotating device slots.  The
 * first copy waits for the work already queued on `stream`; `stream` waits for the last
 * copy, so synchronising `stream` makes every out_host[i] valid. */
DSLASH_API dslash_status dslash_apply_host_batch(dslash_t h, int32_t n, void* const* out_host,
                                                 const void* const* in_host, int32_t parity,
                                                 dslash_stream_t stream);

/* dslash_apply that also hands its output to the next apply (DSLASH_OPT_PUSH; the
 * "compute step followed by an exchange" of D_{p,1-p} D_{1-p,p}).  Every target site within 3
 * slices of a partitioned face stores its result into the neighbour's ghost face as well as
 * into out; the neighbours' ready flags are raised behind the kernel.  The NEXT apply (or
 * halo_start) on this handle, on every rank, must take `out` as its source: it then exchanges
 * no bytes; any other source returns DSLASH_ERR_STATE.  Without a halo it equals dslash_apply.
 * Errors as dslash_apply, plus DSLASH_ERR_STATE without DSLASH_OPT_PUSH. */
DSLASH_API dslash_status dslash_apply_push(dslash_t h, void* out, const void* in, int32_t parity,
                                           dslash_stream_t stream);

/* The even-odd normal operator (the conjugate-gradient step of MILC's
 * su3_rhmd_hisq):  out = A_p in,  A_p = m^2 - D_{p,1-p} D_{1-p,p}, where D_{a,b}
 * is the Dslash from parity b to target parity a.  D is anti-Hermitian, so A_p = m^2 +
 * D_{1-p,p}^dag D_{1-p,p} is Hermitian positive definite for m != 0.  in, out: fp64 [3][Vh]
 * vectors on parity p.  Needs parity_mask DSLASH_BOTH and fp64 vectors (DSLASH_F64 or
 * DSLASH_MIXED; DSLASH_F32 returns DSLASH_ERR_UNSUPPORTED).  Two applies + one fused
 * m^2-subtraction kernel, stream-ordered.  With DSLASH_OPT_PUSH the first apply pushes its
 * output's faces (dslash_apply_push), so the second exchanges no bytes (also inside CG). */
DSLASH_API dslash_status dslash_normal_apply(dslash_t h, void* out, const void* in, int32_t parity, double mass,
                                             dslash_stream_t stream);

/* Conjugate gradient for A_p x = b (A_p as above), starting from x = 0, stopping when
 * |r_k| <= rel_tol |b| or after max_iter iterations.  Dot products are accumulated as
 * double-double sums (per thread, block, GPU and over the ranks in rank order: the per-rank
 * sums are all-gathered with ncclAllGather, or through the P2P transport's IPC-mapped slots when
 * the handle has no communicator) and rounded once, so every rank gets the same bits and a
 * P-rank solve runs the 1-rank iterates bit for bit (unless a sum lies within ~1e-26 relative of
 * a rounding boundary; DESIGN.md §12 f-3).  With one rank the
 * vector work of an iteration (m^2 p - q, both dot products, the x / r / p updates) runs as one
 * cooperative kernel with the same arithmetic and reduction order (bitwise the same iterates).  Synchronous:
 * returns after the solve (it reads each dot product on the host).  iters (may be NULL)
 * receives the iteration count, rel_resid (may be NULL) the TRUE relative residual
 * |b - A x| / |b| recomputed at the end.  Returns DSLASH_ERR_NOT_CONVERGED (not sticky) if the
 * recursive residual did not reach rel_tol. */
DSLASH_API dslash_status dslash_cg(dslash_t h, void* x, const void* b, int32_t parity, double mass, double rel_tol,
                                   int32_t max_iter, int32_t* iters, double* rel_resid, dslash_stream_t stream);

/* Mixed-precision CG by defect correction (QUDA's "mixed precision" solvers):
 * x = 0, r = b; repeat { solve A_p e = r in fp32 (F32 kernels on fp32 links rounded once from
 * the handle's fp64 links, fp32 vectors, fp64 dot products) by CG until |r_e| <= inner_tol |r|;
 * x += e in fp64; r = b - A_p x in fp64 } until |r| <= rel_tol |b| or max_iter inner iterations
 * in total.  The answer is accurate to rel_tol in fp64 (the TRUE residual is what stops it).
 * Needs a DSLASH_F64 handle with parity_mask DSLASH_BOTH and a site / dir2 / dir4 kernel; the
 * fp32 links (half the fp64 link memory) are built on the first call after load_links.
 * 0 < inner_tol < 1.  iters: inner iterations in total; outer_iters: corrections; rel_resid:
 * the final true relative residual (each may be NULL).  Synchronous; DSLASH_ERR_NOT_CONVERGED
 * as dslash_cg. */
DSLASH_API dslash_status dslash_cg_mixed(dslash_t h, void* x, const void* b, int32_t parity, double mass,
                                         double rel_tol, double inner_tol, int32_t max_iter, int32_t* iters,
                                         int32_t* outer_iters, double* rel_resid, dslash_stream_t stream);

/* CG for nrhs <= 8 independent systems A_p x_r = b_r (A_p as dslash_cg) that share every pass over
 * the links (SURVEY.md §8(f)-3 on the §8(f)-4 multi-RHS stencil): each
 * iteration applies the stencil twice to all nrhs directions at once
 * (dslash_apply_multi_blocked), then every system advances on its own scalars
 * (Hestenes-Stiefel, double-double dot products).  A system whose residual met rel_tol is frozen
 * while the others continue.  x, b: device buffers of nrhs x 3 x Vh_local fp64 complex in the
 * SITE-BLOCKED layout (dslash_apply_multi_blocked; dslash_vectors_to_blocked converts).
 * iters[r]: the iteration at which system r converged (max_iter if it did not); rel_resid[r]: its
 * true |b_r - A x_r| / |b_r| (each array nrhs long, or NULL).  Requires a DSLASH_F64 or
 * DSLASH_MIXED handle with parity_mask DSLASH_BOTH, one rank, nonzero mass, the blocked layout's
 * conditions; synchronous; DSLASH_ERR_NOT_CONVERGED (not sticky) if a system did not converge. */
DSLASH_API dslash_status dslash_cg_multi_blocked(dslash_t h, int32_t nrhs, void* x, const void* b, int32_t parity,
                                                 double mass, double rel_tol, int32_t max_iter, int32_t* iters,
                                                 double* rel_resid, dslash_stream_t stream);

/* Halo exchange only: start sending the depth-3 faces of `in` (source parity
 * src_parity) after the work already queued on `stream`; dslash_halo_wait makes
 * `stream` wait for the ghost zones.  No-op when no direction has a halo.  Exposed
 * so callers can overlap their own work; dslash_apply calls both itself. */
DSLASH_API dslash_status dslash_halo_start(dslash_t h, const void* in, int32_t src_parity, dslash_stream_t stream);
DSLASH_API dslash_status dslash_halo_wait(dslash_t h, dslash_stream_t stream);

/* Synchronise the handle's streams and surface asynchronous CUDA/NCCL errors. */
DSLASH_API dslash_status dslash_sync(dslash_t h);

/* Sum of the durations of the kernels of class `which` (DSLASH_TIMING_INTERIOR / _BOUNDARY,
 * or DSLASH_TIMING_ALL for every class) recorded since the last dslash_kernel_timing_reset
 * (DSLASH_OPT_TIMING = 1); synchronises on the recorded events.  Every timed launch keeps
 * one event pair until the next reset. */
DSLASH_API dslash_status dslash_kernel_timing(dslash_t h, int32_t which, double* total_ms, int64_t* launches);
DSLASH_API dslash_status dslash_kernel_timing_reset(dslash_t h);

/* The recorded intervals themselves, in record order (DSLASH_OPT_TIMING = 1): a timeline of
 * kernels and exchanges across the handle's streams (the overlap of the exchange with the
 * interior kernel, without a system profiler).  Writes up to max_entries
 * entries: kinds[i] (DSLASH_TIMING_*), start_ms[i] and end_ms[i] relative to the start of the
 * first recorded interval since the last reset; *n receives the number of entries recorded
 * (may exceed max_entries).  Synchronises on the recorded events.  Host arrays, caller-owned. */
DSLASH_API dslash_status dslash_timeline(dslash_t h, int64_t max_entries, int32_t* kinds, double* start_ms,
                                         double* end_ms, int64_t* n);

/* Copy the plan the handle uses. */
DSLASH_API dslash_status dslash_get_plan(dslash_t h, dslash_plan_t* plan);

/* Number of local target sites per parity (Vh_local), or -1 for a NULL handle. */
DSLASH_API int64_t dslash_local_half_volume(dslash_t h);

/* Release everything the handle owns (synchronises first).  NULL is a no-op. */
DSLASH_API dslash_status dslash_destroy(dslash_t h);

/* Human-readable description of the handle's first error ("" if none); with h = NULL,
 * the last error of a failed dslash_create / dslash_plan in this thread. */
DSLASH_API const char* dslash_error_string(dslash_t h);

#ifdef __cplusplus
}
#endif

#endif /* HISQ_DSLASH_H */
