// dslash_lib.cu -- C ABI of the B200-native HISQ Dslash (include/hisq_dslash.h).
//
// Host runtime: lattice decomposition (dslash_plan), device memory ownership, the depth-3
// halo exchange (NCCL send/recv over NVLink on an internal stream, or device copies when the
// neighbour is this rank), kernel launches and error reporting.  Every step of the Dslash
// itself runs in the kernels of stencil.cuh / links.cuh.
#include <nccl.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "handle.h"
#include "common.cuh"
#include "links.cuh"
#include "stencil.cuh"
#include "dispatch.h"

using namespace hisq;

// ============================================================================ errors
static thread_local std::string g_last_error;

dslash_status hisq_fail(dslash_t h, dslash_status st, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    if (h) {
        if (h->err == DSLASH_OK) {
            h->err = st;
            h->msg = buf;
        }
    } else {
        g_last_error = buf;
    }
    return st;
}
#define fail hisq_fail

// ============================================================================ plan (host only)
extern "C" dslash_status dslash_plan(const int32_t G[4], const int32_t P[4], int32_t rank, int32_t nranks,
                                     int32_t force_halo_mask, dslash_plan_t* out) {
    if (!G || !P || !out) return fail(nullptr, DSLASH_ERR_ARG, "dslash_plan: NULL argument");
    dslash_plan_t p;
    memset(&p, 0, sizeof p);
    int64_t prod = 1;
    for (int d = 0; d < 4; ++d) {
        if (G[d] < 2 || (G[d] & 1))
            return fail(nullptr, DSLASH_ERR_ARG, "global extent %d of dim %d must be even and >= 2", G[d], d);
        if (P[d] < 1) return fail(nullptr, DSLASH_ERR_ARG, "proc_grid[%d] = %d must be >= 1", d, P[d]);
        if (G[d] % P[d])
            return fail(nullptr, DSLASH_ERR_ARG, "global extent %d of dim %d not divisible by proc_grid %d", G[d], d,
                        P[d]);
        prod *= P[d];
    }
    if (P[0] != 1 || P[1] != 1)
        return fail(nullptr, DSLASH_ERR_UNSUPPORTED, "only z and t may be partitioned (proc_grid = {1,1,Pz,Pt})");
    if (prod != nranks) return fail(nullptr, DSLASH_ERR_ARG, "prod(proc_grid) = %lld != nranks = %d", (long long)prod, nranks);
    if (rank < 0 || rank >= nranks) return fail(nullptr, DSLASH_ERR_ARG, "rank %d out of range [0,%d)", rank, nranks);
    if (force_halo_mask & ~0xC)
        return fail(nullptr, DSLASH_ERR_UNSUPPORTED, "halo directions other than z (bit 2) and t (bit 3)");
    p.rank = rank;
    p.nranks = nranks;
    // rank = cx + Px*(cy + Py*(cz + Pz*ct)) with Px = Py = 1
    int r = rank;
    for (int d = 0; d < 4; ++d) {
        p.global_dims[d] = G[d];
        p.proc_grid[d] = P[d];
        p.proc_coords[d] = r % P[d];
        r /= P[d];
        p.local_dims[d] = G[d] / P[d];
        p.origin[d] = p.proc_coords[d] * p.local_dims[d];
    }
    for (int d = 0; d < 4; ++d) {
        p.halo[d] = (P[d] > 1) || ((force_halo_mask >> d) & 1);
        for (int side = 0; side < 2; ++side) {
            int c[4] = {p.proc_coords[0], p.proc_coords[1], p.proc_coords[2], p.proc_coords[3]};
            c[d] = (c[d] + (side ? 1 : P[d] - 1)) % P[d];
            p.nbr_rank[d][side] = c[0] + P[0] * (c[1] + P[1] * (c[2] + P[2] * c[3]));
        }
        if (p.halo[d] && (p.local_dims[d] < 4 || (p.local_dims[d] & 1)))
            return fail(nullptr, DSLASH_ERR_ARG,
                        "local extent %d of halo dim %d must be even and >= 4 (depth-3 halo, parity)",
                        p.local_dims[d], d);
    }
    const int64_t V = (int64_t)p.local_dims[0] * p.local_dims[1] * p.local_dims[2] * p.local_dims[3];
    p.vh_local = V / 2;
    for (int d = 0; d < 4; ++d) p.face_vh[d] = p.halo[d] ? 3 * (V / p.local_dims[d]) / 2 : 0;

    // interior box: [3, L-3) along halo dims, full otherwise
    dslash_box_t full;
    for (int d = 0; d < 4; ++d) {
        full.lo[d] = 0;
        full.hi[d] = p.local_dims[d];
    }
    dslash_box_t in = full;
    bool empty = false;
    for (int d = 0; d < 4; ++d)
        if (p.halo[d]) {
            in.lo[d] = 3;
            in.hi[d] = p.local_dims[d] - 3;
            if (in.lo[d] >= in.hi[d]) empty = true;
        }
    auto count = [](const dslash_box_t& b) {
        int64_t n = (b.hi[0] - b.lo[0]) / 2;
        for (int d = 1; d < 4; ++d) n *= (b.hi[d] - b.lo[d]);
        return n;
    };
    if (empty) {
        p.n_interior = 0;
        p.n_boundary = 1;
        p.boundary[0] = full;
    } else {
        p.n_interior = 1;
        p.interior[0] = in;
        int nb = 0;
        dslash_box_t rest = full;  // region still to be covered: shrinks as slabs are cut off
        for (int d = 3; d >= 2; --d) {
            if (!p.halo[d]) continue;
            dslash_box_t lo = rest, hi = rest;
            lo.hi[d] = 3;
            hi.lo[d] = p.local_dims[d] - 3;
            p.boundary[nb++] = lo;
            p.boundary[nb++] = hi;
            rest.lo[d] = 3;
            rest.hi[d] = p.local_dims[d] - 3;
        }
        p.n_boundary = nb;
    }
    for (int i = 0; i < p.n_interior; ++i) p.interior_sites += count(p.interior[i]);
    for (int i = 0; i < p.n_boundary; ++i) p.boundary_sites += count(p.boundary[i]);
    *out = p;
    return DSLASH_OK;
}

// ============================================================================ handle
extern "C" int32_t dslash_device_count(void) {
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    return n;
}

extern "C" dslash_status dslash_set_device(int32_t device) {
    const int n = dslash_device_count();
    if (device < 0 || device >= n) return fail(nullptr, DSLASH_ERR_ARG, "device %d not in [0, %d)", device, n);
    cudaError_t e = cudaSetDevice(device);
    if (e != cudaSuccess) return fail(nullptr, DSLASH_ERR_CUDA, "cudaSetDevice(%d): %s", device, cudaGetErrorString(e));
    return DSLASH_OK;
}

extern "C" dslash_status dslash_get_unique_id(void* id_out) {
    if (!id_out) return fail(nullptr, DSLASH_ERR_ARG, "NULL id_out");
    ncclUniqueId id;
    ncclResult_t r = ncclGetUniqueId(&id);
    if (r != ncclSuccess) return fail(nullptr, DSLASH_ERR_NCCL, "ncclGetUniqueId: %s", ncclGetErrorString(r));
    memcpy(id_out, &id, sizeof id);
    return DSLASH_OK;
}

static void free_links(dslash_t h) {
    for (int p = 0; p < 2; ++p)
        if (h->links[p]) {
            cudaFree(h->links[p]);
            h->links[p] = nullptr;
        }
    h->loaded = false;
}

// Does direction d's exchange go through NCCL (or, under the P2P transport, the peers)?  A
// neighbour on another rank always does; a self-neighbour (P_d = 1 with FORCE_HALO) is served by
// device copies unless DSLASH_OPT_SELF_NCCL routes it through NCCL send/recv to this rank, the
// message pattern of P_d = 2 (both neighbours one peer, messages matched in issue order).
static bool exch_remote(const dslash_s* h, int d) {
    return h->plan.nbr_rank[d][0] != h->plan.rank || h->self_nccl;
}

static void free_halo(dslash_t h) {
    for (int d = 0; d < 4; ++d)
        for (int s = 0; s < 2; ++s)
            if (h->ghost[d][s]) {
                cudaFree(h->ghost[d][s]);
                h->ghost[d][s] = nullptr;
            }
    for (int s = 0; s < 2; ++s)
        if (h->zsend[s]) {
            cudaFree(h->zsend[s]);
            h->zsend[s] = nullptr;
        }
}

static dslash_status alloc_halo(dslash_t h, int nrhs) {
    free_halo(h);
    const dslash_plan_t& p = h->plan;
    const size_t es = h->precision == DSLASH_F32 ? 8 : 16;
    for (int d = 2; d < 4; ++d) {
        h->ghost_bank[d] = 0;
        if (!p.halo[d]) continue;
        // producer push: two banks, so an apply can push the next apply's faces into one while
        // its own boundary kernel (and the neighbours') still read the other
        const size_t bank = (size_t)nrhs * 3 * p.face_vh[d] * es;
        if (h->push) h->ghost_bank[d] = bank;
        for (int s = 0; s < 2; ++s) CU(h, cudaMalloc(&h->ghost[d][s], h->push ? 2 * bank : bank));
    }
    if (p.halo[2] && exch_remote(h, 2))
        for (int s = 0; s < 2; ++s) CU(h, cudaMalloc(&h->zsend[s], (size_t)nrhs * 3 * p.face_vh[2] * es));
    h->ghost_rhs = nrhs;
    return DSLASH_OK;
}

static constexpr int kP2PMaxRhs = 8;  // ghost capacity with the P2P transport (IPC-exported once)

// the P2P control block (epoch flags, reduction slots; handle.h P2PControl)
static dslash_status alloc_flags(dslash_t h) {
    if (!h->ctl) {
        CU(h, cudaMalloc(&h->ctl, sizeof(P2PControl)));
        CU(h, cudaMemset(h->ctl, 0, sizeof(P2PControl)));
        h->flags = h->ctl->flags;
    }
    return DSLASH_OK;
}

// bytes of ONE kind (fat or long) of the 3 canonical link slices below the local origin in
// direction d (the link halo of load_links)
static size_t link_slab_bytes(const dslash_plan_t& p, int d) {
    const int64_t V = 2 * p.vh_local;
    return (size_t)3 * (V / p.local_dims[d]) * 36 * sizeof(double2);
}

// P2P: the link-slab receive buffers ([fat | long]) of the halo directions whose minus neighbour
// is another rank; IPC-exported with the ghosts, so they exist before dslash_get_ipc_blob
static dslash_status alloc_lslab(dslash_t h) {
    const dslash_plan_t& p = h->plan;
    for (int d = 2; d < 4; ++d) {
        if (!p.halo[d] || p.nbr_rank[d][0] == p.rank || h->lslab[d]) continue;
        h->lslab_bytes[d] = link_slab_bytes(p, d);
        CU(h, cudaMalloc(&h->lslab[d], 2 * h->lslab_bytes[d]));
    }
    return DSLASH_OK;
}

extern "C" dslash_status dslash_create(const int32_t G[4], const int32_t P[4], int32_t parity_mask, int32_t precision,
                                       const void* nccl_unique_id, int32_t nranks, int32_t rank, dslash_t* out) {
    if (!out) return fail(nullptr, DSLASH_ERR_ARG, "NULL out");
    *out = nullptr;
    if (parity_mask < DSLASH_EVEN || parity_mask > DSLASH_BOTH)
        return fail(nullptr, DSLASH_ERR_ARG, "parity_mask %d not in {0,1,2}", parity_mask);
    if (precision != DSLASH_F64 && precision != DSLASH_F32 && precision != DSLASH_MIXED)
        return fail(nullptr, DSLASH_ERR_ARG, "precision %d unknown", precision);
    dslash_plan_t plan;
    dslash_status st = dslash_plan(G, P, rank, nranks, 0, &plan);
    if (st != DSLASH_OK) return st;
    dslash_t h = new dslash_s();
    h->plan = plan;
    memcpy(h->global_dims, G, sizeof h->global_dims);
    memcpy(h->proc_grid, P, sizeof h->proc_grid);
    h->parity_mask = parity_mask;
    h->precision = precision;
    auto bail = [&](dslash_status s) {
        g_last_error = h->msg;
        dslash_destroy(h);
        return s;
    };
    cudaError_t e = cudaGetDevice(&h->device);
    if (e != cudaSuccess) {
        fail(h, DSLASH_ERR_CUDA, "cudaGetDevice: %s", cudaGetErrorString(e));
        return bail(DSLASH_ERR_CUDA);
    }
    // the exchange and the boundary kernel (queued behind it on the same stream) get the greatest
    // stream priority: their blocks are dispatched ahead of the interior kernel's pending blocks
    // once their inputs are ready
    int prio_lo = 0, prio_hi = 0;
    cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
    if ((e = cudaStreamCreateWithPriority(&h->comm, cudaStreamNonBlocking, prio_hi)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&h->ev_bdone, cudaEventDisableTiming)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&h->ev_start, cudaEventDisableTiming)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&h->ev_halo, cudaEventDisableTiming)) != cudaSuccess) {
        fail(h, DSLASH_ERR_CUDA, "stream/event creation: %s", cudaGetErrorString(e));
        return bail(DSLASH_ERR_CUDA);
    }
    h->transport = (nranks > 1 && !nccl_unique_id) ? DSLASH_TRANSPORT_P2P : DSLASH_TRANSPORT_NCCL;
    if (nccl_unique_id) {  // nranks == 1: a one-rank communicator (DSLASH_OPT_SELF_NCCL, solver sums)
        ncclUniqueId id;
        memcpy(&id, nccl_unique_id, sizeof id);
        ncclResult_t r = ncclCommInitRank(&h->nccl, nranks, id, rank);
        if (r != ncclSuccess) {
            h->nccl = nullptr;
            fail(h, DSLASH_ERR_NCCL, "ncclCommInitRank: %s", ncclGetErrorString(r));
            return bail(DSLASH_ERR_NCCL);
        }
    }
    if ((st = alloc_halo(h, h->transport == DSLASH_TRANSPORT_P2P ? kP2PMaxRhs : 1)) != DSLASH_OK) return bail(st);
    if (h->transport == DSLASH_TRANSPORT_P2P && (st = alloc_flags(h)) != DSLASH_OK) return bail(st);
    *out = h;
    return DSLASH_OK;
}

extern "C" dslash_status dslash_set_option(dslash_t h, int32_t key, int64_t value) {
    DeviceGuard device_guard(h);
    if (!h) return fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    switch (key) {
        case DSLASH_OPT_KERNEL:
            if (value != DSLASH_KERNEL_SITE && value != DSLASH_KERNEL_DIR4 && value != DSLASH_KERNEL_DIR2)
                return fail(h, DSLASH_ERR_ARG, "unknown kernel variant %lld", (long long)value);
            if (h->loaded && value != h->kernel)
                return fail(h, DSLASH_ERR_STATE, "kernel variant fixes the link layout: set it before load_links");
            if (h->stage && value != DSLASH_KERNEL_SITE && value != DSLASH_KERNEL_DIR2)
                return fail(h, DSLASH_ERR_UNSUPPORTED, "the neighbour-staged kernel serves the site and dir2 variants");
            h->kernel = (int)value;
            return DSLASH_OK;
        case DSLASH_OPT_BLOCK:
            if (value != 0 && (value < 32 || value > 256 || (value & 31)))
                return fail(h, DSLASH_ERR_ARG, "block size %lld must be 0 or a multiple of 32 in [32,256]",
                            (long long)value);
            h->block = (int)value;
            return DSLASH_OK;
        case DSLASH_OPT_FORCE_HALO: {
            if (h->loaded || h->p2p_ready)
                return fail(h, DSLASH_ERR_STATE, "FORCE_HALO must be set before load_links and the IPC setup");
            dslash_plan_t p;
            dslash_status st = dslash_plan(h->global_dims, h->proc_grid, h->plan.rank, h->plan.nranks, (int)value, &p);
            if (st != DSLASH_OK) return fail(h, st, "%s", g_last_error.c_str());
            h->plan = p;
            h->force_halo = (int)value;
            return alloc_halo(h, h->transport == DSLASH_TRANSPORT_P2P ? kP2PMaxRhs : 1);
        }
        case DSLASH_OPT_SELF_NCCL: {
            if (h->loaded || h->p2p_ready)
                return fail(h, DSLASH_ERR_STATE, "SELF_NCCL must be set before load_links");
            if (value && (h->transport != DSLASH_TRANSPORT_NCCL || !h->nccl))
                return fail(h, DSLASH_ERR_STATE,
                            "SELF_NCCL needs the NCCL transport and a communicator (dslash_create with an id)");
            h->self_nccl = value != 0;
            return alloc_halo(h, 1);
        }
        case DSLASH_OPT_HALO_DRYRUN:
            if (value && h->transport != DSLASH_TRANSPORT_NCCL)
                return fail(h, DSLASH_ERR_UNSUPPORTED, "HALO_DRYRUN serves the NCCL / device-copy transport");
            h->halo_dryrun = value != 0;
            return DSLASH_OK;
        case DSLASH_OPT_STAGE:
            if (value && h->kernel != DSLASH_KERNEL_SITE && h->kernel != DSLASH_KERNEL_DIR2)
                return fail(h, DSLASH_ERR_UNSUPPORTED, "the neighbour-staged kernel serves the site and dir2 variants");
            if (value && h->precision == DSLASH_F32 && (h->plan.local_dims[0] / 2) % 2)
                return fail(h, DSLASH_ERR_UNSUPPORTED, "staged fp32 rows need Lx/2 even (16-byte bulk copies)");
            h->stage = value != 0;
            return DSLASH_OK;
        case DSLASH_OPT_OVERLAP:
            if (value < 0 || value > DSLASH_OVERLAP_DIRS)
                return fail(h, DSLASH_ERR_ARG, "overlap mode %lld not in {0, 1, 2}", (long long)value);
            h->overlap = (int)value;
            return DSLASH_OK;
        case DSLASH_OPT_TIMING:
            h->timing = value != 0;
            return DSLASH_OK;
        case DSLASH_OPT_TRANSPORT: {
            if (value != DSLASH_TRANSPORT_NCCL && value != DSLASH_TRANSPORT_P2P)
                return fail(h, DSLASH_ERR_ARG, "unknown transport %lld", (long long)value);
            if (h->loaded || h->p2p_ready)
                return fail(h, DSLASH_ERR_STATE, "the transport must be chosen before load_links / IPC setup");
            if (value == DSLASH_TRANSPORT_NCCL && h->plan.nranks > 1 && !h->nccl)
                return fail(h, DSLASH_ERR_STATE, "NCCL transport needs dslash_create with an NCCL unique id");
            h->transport = (int)value;
            if (value != DSLASH_TRANSPORT_P2P) h->push = 0;
            dslash_status st = alloc_halo(h, value == DSLASH_TRANSPORT_P2P ? kP2PMaxRhs : 1);
            if (st == DSLASH_OK && value == DSLASH_TRANSPORT_P2P) st = alloc_flags(h);
            return st;
        }
        case DSLASH_OPT_PDL:
            h->pdl = value != 0;
            return DSLASH_OK;
        case DSLASH_OPT_LONG_RECON:
            if (value != 18 && value != 12 && value != 9)
                return fail(h, DSLASH_ERR_ARG, "long-link recon %lld must be 18, 12 or 9", (long long)value);
            if (h->loaded && value != h->recon)
                return fail(h, DSLASH_ERR_STATE, "long-link recon fixes the link layout: set it before load_links");
            h->recon = (int)value;
            return DSLASH_OK;
        case DSLASH_OPT_PUSH: {
            if (h->loaded || h->p2p_ready)
                return fail(h, DSLASH_ERR_STATE, "PUSH must be set before load_links and the IPC setup");
            if (value && h->transport != DSLASH_TRANSPORT_P2P)
                return fail(h, DSLASH_ERR_UNSUPPORTED, "the producer push needs the P2P transport (peer-mapped ghosts)");
            h->push = value != 0;
            h->pushed_epoch = 0;
            h->pushed_src = nullptr;
            return alloc_halo(h, kP2PMaxRhs);
        }
        case DSLASH_OPT_MIN_BLOCKS:
            if (value != 0 && (value < 2 || value > 4))
                return fail(h, DSLASH_ERR_ARG, "min_blocks %lld must be 0, 2, 3 or 4", (long long)value);
            h->min_blocks = (int)value;
            return DSLASH_OK;
        default:
            return fail(h, DSLASH_ERR_ARG, "unknown option %d", key);
    }
}

// bytes of one complex element of the vectors / of the stored links
static size_t vec_elem(const dslash_s* h) { return h->precision == DSLASH_F32 ? 8 : 16; }
static size_t link_elem(const dslash_s* h) { return h->precision == DSLASH_F64 ? 16 : 8; }

static int lanes_of(int kernel) {
    return kernel == DSLASH_KERNEL_DIR4 ? 4 : kernel == DSLASH_KERNEL_DIR2 ? 2 : 1;
}

typedef int (*WriteValue32Fn)(cudaStream_t, unsigned long long, unsigned int, unsigned int);
typedef int (*WaitValue32Fn)(cudaStream_t, unsigned long long, unsigned int, unsigned int);
static WriteValue32Fn write_value_fn();
static WaitValue32Fn wait_value_fn();
static dslash_status p2p_prepare(dslash_t h);

// ============================================================================ link loading
// slab_fat / slab_lng (may be NULL): caller-provided lower link slabs per direction (same device-ness
// as fat / lng); where absent for a halo direction with another rank as neighbour, NCCL fetches them
static dslash_status load_links_impl(dslash_t h, const void* fat, const void* lng, const void* const* slab_fat_in,
                                     const void* const* slab_lng_in, int32_t on_device, dslash_stream_t stream) {
    DeviceGuard device_guard(h);
    if (!h) return fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    if (!fat || !lng) return fail(h, DSLASH_ERR_ARG, "NULL link pointer");
    cudaStream_t s = (cudaStream_t)stream;
    const dslash_plan_t& p = h->plan;
    const int64_t V = 2 * p.vh_local;
    const size_t canon_bytes = (size_t)V * 36 * sizeof(double2);
    std::vector<void*> tmp;
    // P2P link halo (below): directions whose slab arrives in h->lslab, and the epoch of this load
    bool p2p_link[4] = {false, false, false, false};
    unsigned int le = 0;
    bool p2p_released = false;
    // my slab buffers are consumed (or this load failed after the exchange): release them to my
    // minus neighbours, so their next load_links does not wait forever
    auto release_p2p = [&]() -> bool {
        if (!le || p2p_released) return true;
        p2p_released = true;
        WriteValue32Fn wr = write_value_fn();
        for (int d = 3; d >= 2; --d)
            if (p2p_link[d] && wr((cudaStream_t)stream,
                                  (unsigned long long)(uintptr_t)(h->peer_ctl[h->plan.nbr_rank[d][0]]->flags + 20 + d),
                                  le, 0) != 0)
                return false;
        return true;
    };
    auto cleanup = [&]() {
        release_p2p();
        for (void* q : tmp) cudaFree(q);
    };
#define CUL(call)                                                                                     \
    do {                                                                                              \
        cudaError_t e_ = (call);                                                                      \
        if (e_ != cudaSuccess) {                                                                      \
            cudaStreamSynchronize(s);                                                                 \
            cleanup();                                                                                \
            return fail(h, e_ == cudaErrorMemoryAllocation ? DSLASH_ERR_OOM : DSLASH_ERR_CUDA,        \
                        "%s:%d %s: %s", __FILE__, __LINE__, #call, cudaGetErrorString(e_));           \
        }                                                                                             \
    } while (0)
    const double2* dfat = (const double2*)fat;
    const double2* dlng = (const double2*)lng;
    if (!on_device) {
        void *a, *b;
        CUL(cudaMalloc(&a, canon_bytes));
        tmp.push_back(a);
        CUL(cudaMalloc(&b, canon_bytes));
        tmp.push_back(b);
        CUL(cudaMemcpyAsync(a, fat, canon_bytes, cudaMemcpyHostToDevice, s));
        CUL(cudaMemcpyAsync(b, lng, canon_bytes, cudaMemcpyHostToDevice, s));
        dfat = (const double2*)a;
        dlng = (const double2*)b;
    }
    // lower link slabs: the 3 slices just below the local origin in each halo direction
    LinkConvParams C{};
    C.fat = dfat;
    C.lng = dlng;
    for (int d = 0; d < 4; ++d) C.L[d] = p.local_dims[d];
    C.lxh = p.local_dims[0] / 2;
    C.vh = p.vh_local;
    C.lanes = lanes_of(h->kernel);
    C.recon = h->recon;
    C.paired = h->precision != DSLASH_F64;
    int halo_mask = 0;
    for (int d = 2; d < 4; ++d)
        if (p.halo[d]) halo_mask |= 1 << d;
    C.halo_mask = halo_mask;
    double2* slab[4][2] = {};   // [mu][fat/long] received
    double2* send[4][2] = {};   // packed top slabs (z, NCCL only)
    // Exchange: rank sends its top 3 slices to its plus neighbour, receives into its lower
    // slab from its minus neighbour.  All ranks issue t then z, fat then long (same order).
    // NCCL transport: ncclSend / ncclRecv.  P2P transport: the slices are copied straight into
    // the plus neighbour's IPC-mapped slab buffer (p2p_link), ordered by epoch flags.
    bool need_nccl = false;
    bool given[4] = {false, false, false, false};
    for (int d = 3; d >= 2; --d) {
        if (!p.halo[d]) continue;
        given[d] = slab_fat_in && slab_lng_in && slab_fat_in[d] && slab_lng_in[d];
        if (given[d] || !exch_remote(h, d)) continue;
        if (h->transport == DSLASH_TRANSPORT_P2P)
            p2p_link[d] = true;
        else
            need_nccl = true;
    }
    for (int d = 2; d < 4; ++d) {
        if (!p.halo[d]) continue;
        if (p2p_link[d]) {   // received in place, in the library-owned IPC-exported buffer
            if (!h->lslab[d]) {
                cleanup();
                return fail(h, DSLASH_ERR_STATE, "P2P link halo: call dslash_get_ipc_blob / dslash_open_ipc_blobs first");
            }
            slab[d][0] = (double2*)h->lslab[d];
            slab[d][1] = (double2*)(h->lslab[d] + h->lslab_bytes[d]);
            continue;
        }
        const int64_t slab_elems = 3 * (V / p.local_dims[d]) * 36;
        for (int k = 0; k < 2; ++k) {
            CUL(cudaMalloc(&slab[d][k], slab_elems * sizeof(double2)));
            tmp.push_back(slab[d][k]);
        }
    }
    if (need_nccl && !h->nccl) {
        cleanup();
        return fail(h, DSLASH_ERR_STATE,
                    "no NCCL communicator for the link halo: pass the slabs with dslash_load_links_halo");
    }
    const int L0 = p.local_dims[0], L1 = p.local_dims[1], L2 = p.local_dims[2], L3 = p.local_dims[3];
    const size_t row = (size_t)L0 * L1 * 36 * sizeof(double2);  // one z-slice of one t
    for (int d = 3; d >= 2; --d) {
        if (!p.halo[d]) continue;
        if (given[d]) {
            const size_t bytes = (size_t)3 * (V / p.local_dims[d]) * 36 * sizeof(double2);
            const cudaMemcpyKind kind = on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
            CUL(cudaMemcpyAsync(slab[d][0], slab_fat_in[d], bytes, kind, s));
            CUL(cudaMemcpyAsync(slab[d][1], slab_lng_in[d], bytes, kind, s));
            continue;
        }
        if (p2p_link[d]) continue;   // below
        for (int k = 0; k < 2; ++k) {
            const double2* src = k ? dlng : dfat;
            if (d == 3) {
                const double2* top = src + (size_t)(L3 - 3) * L2 * L1 * L0 * 36;
                if (!exch_remote(h, 3))
                    CUL(cudaMemcpyAsync(slab[3][k], top, 3 * (size_t)L2 * row, cudaMemcpyDeviceToDevice, s));
                else
                    send[3][k] = (double2*)top;  // contiguous: zero copy
            } else {
                double2* dst = slab[2][k];
                if (exch_remote(h, 2)) {
                    CUL(cudaMalloc(&send[2][k], 3 * (size_t)L3 * row));
                    tmp.push_back(send[2][k]);
                    dst = send[2][k];
                }
                // [t][z in L2-3..L2-1][y][x] -> [t][d][y][x]
                CUL(cudaMemcpy2DAsync(dst, 3 * row, src + (size_t)(L2 - 3) * L1 * L0 * 36, (size_t)L2 * row, 3 * row,
                                      L3, cudaMemcpyDeviceToDevice, s));
            }
        }
    }
    if (need_nccl) {
        CUL(cudaStreamSynchronize(s));
        ncclResult_t r = ncclGroupStart();
        for (int d = 3; d >= 2 && r == ncclSuccess; --d) {
            if (!p.halo[d] || !exch_remote(h, d) || given[d]) continue;
            const size_t n = (size_t)3 * (V / p.local_dims[d]) * 36 * 2;  // doubles
            for (int k = 0; k < 2 && r == ncclSuccess; ++k) {
                r = ncclSend(send[d][k], n, ncclDouble, p.nbr_rank[d][1], h->nccl, s);
                if (r == ncclSuccess) r = ncclRecv(slab[d][k], n, ncclDouble, p.nbr_rank[d][0], h->nccl, s);
            }
        }
        ncclResult_t r2 = ncclGroupEnd();
        if (r == ncclSuccess) r = r2;
        if (r != ncclSuccess) {
            cleanup();
            return fail(h, DSLASH_ERR_NCCL, "link halo exchange: %s", ncclGetErrorString(r));
        }
    }
    // P2P link halo of epoch e: wait until my plus neighbour converted what I sent at e - 1,
    // copy my top slices into its buffer, raise its lslab_ready; then wait for my minus
    // neighbour's (all ranks send before they wait: no cycle of waits).  Released after the
    // conversion below.
    const bool any_p2p = p2p_link[2] || p2p_link[3];
    if (any_p2p) {
        dslash_status pst = p2p_prepare(h);
        WriteValue32Fn wr = write_value_fn();
        WaitValue32Fn wt = wait_value_fn();
        if (pst == DSLASH_OK && (!wr || !wt)) pst = fail(h, DSLASH_ERR_UNSUPPORTED, "stream memory operations unavailable");
        if (pst != DSLASH_OK) {
            cleanup();
            return pst;
        }
        le = ++h->link_epoch;
        for (int d = 3; d >= 2; --d) {
            if (!p2p_link[d]) continue;
            const int plus = p.nbr_rank[d][1];
            if (wt(s, (unsigned long long)(uintptr_t)(h->flags + 20 + d), le - 1, 0) != 0) {
                cleanup();
                return fail(h, DSLASH_ERR_CUDA, "cuStreamWaitValue32 (link slab free) failed");
            }
            for (int k = 0; k < 2; ++k) {
                const double2* src = k ? dlng : dfat;
                char* dst = h->peer_lslab[d] + k * h->lslab_bytes[d];
                if (d == 3)
                    CUL(cudaMemcpyAsync(dst, src + (size_t)(L3 - 3) * L2 * L1 * L0 * 36, 3 * (size_t)L2 * row,
                                        cudaMemcpyDeviceToDevice, s));
                else  // [t][z in L2-3..L2-1][y][x] -> [t][d][y][x]
                    CUL(cudaMemcpy2DAsync(dst, 3 * row, src + (size_t)(L2 - 3) * L1 * L0 * 36, (size_t)L2 * row,
                                          3 * row, L3, cudaMemcpyDeviceToDevice, s));
            }
            if (wr(s, (unsigned long long)(uintptr_t)(h->peer_ctl[plus]->flags + 16 + d), le, 0) != 0) {
                cleanup();
                return fail(h, DSLASH_ERR_CUDA, "cuStreamWriteValue32 (link slab ready) failed");
            }
        }
        for (int d = 3; d >= 2; --d)
            if (p2p_link[d] && wt(s, (unsigned long long)(uintptr_t)(h->flags + 16 + d), le, 0) != 0) {
                cleanup();
                return fail(h, DSLASH_ERR_CUDA, "cuStreamWaitValue32 (link slab ready) failed");
            }
    }
    for (int d = 0; d < 4; ++d) {
        C.slab_fat[d] = slab[d][0];
        C.slab_lng[d] = slab[d][1];
    }
    if (h->recon == 9) {
        // s from the first local long link: |det(s e^{i psi} W)| = s^3
        double2 A[9];
        CUL(cudaMemcpyAsync(A, dlng, sizeof A, cudaMemcpyDeviceToHost, s));
        CUL(cudaStreamSynchronize(s));
        auto cm = [](double2 a, double2 b) { return make_double2(a.x * b.x - a.y * b.y, a.x * b.y + a.y * b.x); };
        auto sub = [](double2 a, double2 b) { return make_double2(a.x - b.x, a.y - b.y); };
        const double2 m0 = sub(cm(A[4], A[8]), cm(A[5], A[7]));
        const double2 m1 = sub(cm(A[3], A[8]), cm(A[5], A[6]));
        const double2 m2 = sub(cm(A[3], A[7]), cm(A[4], A[6]));
        const double2 d0 = cm(A[0], m0), d1 = cm(A[1], m1), d2 = cm(A[2], m2);
        const double sc = std::cbrt(std::hypot(d0.x - d1.x + d2.x, d0.y - d1.y + d2.y));
        if (!(sc > 0.0) || !std::isfinite(sc)) {
            cleanup();
            return fail(h, DSLASH_ERR_ARG, "recon-9: first long link has zero determinant");
        }
        unsigned long long* dmax;
        CUL(cudaMalloc(&dmax, sizeof *dmax));
        tmp.push_back(dmax);
        CUL(cudaMemsetAsync(dmax, 0, sizeof *dmax, s));
        auto check = [&](const double2* arr, int64_t nmat) {
            if (nmat > 0) recon9_check_kernel<<<(unsigned)((nmat + 255) / 256), 256, 0, s>>>(arr, nmat, sc, dmax);
        };
        check(dlng, V * 4);
        for (int d = 2; d < 4; ++d)
            if (slab[d][1]) check(slab[d][1], 3 * (V / p.local_dims[d]) * 4);
        CUL(cudaGetLastError());
        unsigned long long bits = 0;
        CUL(cudaMemcpyAsync(&bits, dmax, sizeof bits, cudaMemcpyDeviceToHost, s));
        CUL(cudaStreamSynchronize(s));
        double err;
        memcpy(&err, &bits, sizeof err);
        // The rebuild divides by n = |a2|^2 + |a3|^2 (stencil.cuh reconstruct_9), so its worst-link
        // error grows with the number of links: the 21 M long links of a random 48^4 lattice reach
        // 1.8e-12 s (32^4: below 1e-12 s).  A link entry off by 1e-11 s moves a Dslash component by
        // at most ~1e-11 s |psi|, i.e. ~1e-14 of max|chi| for these fields: far inside the 1e-12
        // normwise bar, while a wrong parameterisation (not s e^{i psi} SU(3)) is off by O(s).
        if (!(err <= 1e-11 * sc)) {
            cleanup();
            return fail(h, DSLASH_ERR_ARG,
                        "recon-9: long links are not s*e^{i psi}*SU(3) with one real s = %.17g, or lie near the "
                        "parameterisation's singular set (max deviation %.3e)", sc, err);
        }
        h->long_scale = sc;
        h->long_inv_scale = 1.0 / sc;
        C.s9 = sc;
    }
    if (h->recon == 12) {
        // s from the first local long link: det(s W) = s^3
        double2 A[9];
        CUL(cudaMemcpyAsync(A, dlng, sizeof A, cudaMemcpyDeviceToHost, s));
        CUL(cudaStreamSynchronize(s));
        auto cm = [](double2 a, double2 b) { return make_double2(a.x * b.x - a.y * b.y, a.x * b.y + a.y * b.x); };
        auto sub = [](double2 a, double2 b) { return make_double2(a.x - b.x, a.y - b.y); };
        const double2 m0 = sub(cm(A[4], A[8]), cm(A[5], A[7]));
        const double2 m1 = sub(cm(A[3], A[8]), cm(A[5], A[6]));
        const double2 m2 = sub(cm(A[3], A[7]), cm(A[4], A[6]));
        const double det = cm(A[0], m0).x - cm(A[1], m1).x + cm(A[2], m2).x;
        const double sc = std::cbrt(det);
        if (!(std::fabs(sc) > 0.0)) {
            cleanup();
            return fail(h, DSLASH_ERR_ARG, "recon-12: first long link has zero determinant");
        }
        unsigned long long* dmax;
        CUL(cudaMalloc(&dmax, sizeof *dmax));
        tmp.push_back(dmax);
        CUL(cudaMemsetAsync(dmax, 0, sizeof *dmax, s));
        auto check = [&](const double2* arr, int64_t nmat) {
            if (nmat > 0) recon_check_kernel<<<(unsigned)((nmat + 255) / 256), 256, 0, s>>>(arr, nmat, 1.0 / sc, dmax);
        };
        check(dlng, V * 4);
        for (int d = 2; d < 4; ++d)
            if (slab[d][1]) check(slab[d][1], 3 * (V / p.local_dims[d]) * 4);
        CUL(cudaGetLastError());
        unsigned long long bits = 0;
        CUL(cudaMemcpyAsync(&bits, dmax, sizeof bits, cudaMemcpyDeviceToHost, s));
        CUL(cudaStreamSynchronize(s));
        double err;
        memcpy(&err, &bits, sizeof err);
        const double tol = (h->precision == DSLASH_F64 ? 1e-12 : 1e-6) * std::fabs(sc);
        if (!(err <= tol)) {
            cleanup();
            return fail(h, DSLASH_ERR_ARG,
                        "recon-12: long links are not s*SU(3) with one real s = %.17g (max row-2 deviation %.3e)", sc, err);
        }
        h->long_inv_scale = 1.0 / sc;
    }
    // complex entries per target site: 4 mu x (18 fat + long: 18 / 12 / recon-9 8 + the psi entry;
    // the fp32 paired layout gives the psi pair a whole float4)
    const int r9_entries = h->precision == DSLASH_F64 ? 108 : 112;
    const size_t link_bytes =
        (size_t)p.vh_local * (h->recon == 12 ? 120 : h->recon == 9 ? r9_entries : 144) * link_elem(h);
    for (int par = 0; par < 2; ++par)  // a recon change alters the size: reallocate
        if (h->links[par] && h->link_bytes != link_bytes) {
            cudaFree(h->links[par]);
            h->links[par] = nullptr;
        }
    h->link_bytes = link_bytes;
    for (int par = 0; par < 2; ++par) {
        const bool want = h->parity_mask == DSLASH_BOTH || h->parity_mask == par;
        if (!want) continue;
        if (!h->links[par]) CUL(cudaMalloc(&h->links[par], link_bytes));
        C.links = h->links[par];
        C.parity = par;  // origin sum is even, so local and global parity agree
        const int64_t n = p.vh_local * 16;
        const int bs = 256;
        if (h->precision == DSLASH_F64)
            convert_links_kernel<double><<<(unsigned)((n + bs - 1) / bs), bs, 0, s>>>(C);
        else
            convert_links_kernel<float><<<(unsigned)((n + bs - 1) / bs), bs, 0, s>>>(C);
        CUL(cudaGetLastError());
    }
    if (!release_p2p()) {
        cleanup();
        return fail(h, DSLASH_ERR_CUDA, "cuStreamWriteValue32 (link slab free) failed");
    }
    CUL(cudaStreamSynchronize(s));
    cleanup();
#undef CUL
    for (void*& l32 : h->links32)  // the mixed-precision solver's fp32 copies are stale now
        if (l32) {
            cudaFree(l32);
            l32 = nullptr;
        }
    h->loaded = true;
    return DSLASH_OK;
}

extern "C" dslash_status dslash_load_links(dslash_t h, const void* fat, const void* lng, int32_t on_device,
                                           dslash_stream_t stream) {
    return load_links_impl(h, fat, lng, nullptr, nullptr, on_device, stream);
}

// the mixed-precision solver's fp32 links of `parity` (solver.cu need_sloppy): the fp64 internal
// links rounded into the fp32 paired layout of the same lane mapping
dslash_status hisq_convert_links_sloppy(dslash_t h, int parity) {
    const dslash_plan_t& p = h->plan;
    LinkConvParams S{};
    for (int d = 0; d < 4; ++d) S.L[d] = p.local_dims[d];
    S.lxh = p.local_dims[0] / 2;
    S.vh = p.vh_local;
    S.lanes = lanes_of(h->kernel);
    S.recon = h->recon;
    S.s9 = h->long_scale;
    S.paired = 0;
    S.parity = parity;
    S.links = h->links[parity];
    LinkConvParams D = S;
    D.paired = 1;
    if (h->recon == 9) D.recon = 18;  // the fp32 kernels take recon-9 links rebuilt in full
    D.links = h->links32[parity];
    const int64_t n = p.vh_local * 16;
    convert_internal_kernel<<<(unsigned)((n + 255) / 256), 256>>>(S, D);
    CU(h, cudaGetLastError());
    CU(h, cudaDeviceSynchronize());
    return DSLASH_OK;
}

extern "C" dslash_status dslash_get_links(dslash_t h, int32_t parity, void* out_host) {
    DeviceGuard device_guard(h);
    if (!h) return fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    if (!out_host || (parity & ~1)) return fail(h, DSLASH_ERR_ARG, "NULL output or bad parity");
    if (!h->loaded || !h->links[parity]) return fail(h, DSLASH_ERR_STATE, "links of parity %d not loaded", parity);
    const dslash_plan_t& p = h->plan;
    LinkConvParams C{};
    C.links = h->links[parity];
    C.vh = p.vh_local;
    C.lanes = lanes_of(h->kernel);
    C.recon = h->recon;
    C.s9 = h->long_scale;
    C.paired = h->precision != DSLASH_F64;
    const size_t bytes = (size_t)p.vh_local * 144 * sizeof(double2);
    void* tmp = nullptr;
    CU(h, cudaMalloc(&tmp, bytes));
    const int64_t n = p.vh_local * 16;
    if (h->precision == DSLASH_F64)
        export_links_kernel<double><<<(unsigned)((n + 255) / 256), 256>>>(C, (double2*)tmp);
    else
        export_links_kernel<float><<<(unsigned)((n + 255) / 256), 256>>>(C, (double2*)tmp);
    cudaError_t e = cudaGetLastError();
    if (e == cudaSuccess) e = cudaMemcpy(out_host, tmp, bytes, cudaMemcpyDeviceToHost);
    cudaFree(tmp);
    if (e != cudaSuccess) return fail(h, DSLASH_ERR_CUDA, "dslash_get_links: %s", cudaGetErrorString(e));
    return DSLASH_OK;
}

extern "C" dslash_status dslash_load_links_halo(dslash_t h, const void* fat, const void* lng,
                                                const void* const slab_fat[4], const void* const slab_lng[4],
                                                int32_t on_device, dslash_stream_t stream) {
    if (!h) return fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    if (!slab_fat || !slab_lng) return fail(h, DSLASH_ERR_ARG, "NULL slab arrays");
    for (int d = 2; d < 4; ++d)
        if (h->plan.halo[d] && h->plan.nbr_rank[d][1] != h->plan.rank && (!slab_fat[d] || !slab_lng[d]))
            return fail(h, DSLASH_ERR_ARG, "missing link slab for halo direction %d", d);
    return load_links_impl(h, fat, lng, slab_fat, slab_lng, on_device, stream);
}

// cuStreamWriteValue32 through the runtime's driver entry point (no link-time libcuda): a stream's
// front end writes the P2P epoch flags (ready / free), without an SM.
static WriteValue32Fn write_value_fn() {
    static WriteValue32Fn fn = nullptr;
    static bool tried = false;
    if (!tried) {
        tried = true;
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuStreamWriteValue32", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (WriteValue32Fn)p;
        else
            cudaGetLastError();
    }
    return fn;
}

// cuStreamWaitValue32 (flags 0 = CU_STREAM_WAIT_VALUE_GEQ: wait until (int32)(*addr - value) >= 0)
static WaitValue32Fn wait_value_fn() {
    static WaitValue32Fn fn = nullptr;
    static bool tried = false;
    if (!tried) {
        tried = true;
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuStreamWaitValue32", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (WaitValue32Fn)p;
        else
            cudaGetLastError();
    }
    return fn;
}


// ---------------------------------------------------------------------------- P2P transport
struct IpcBlob {
    int32_t magic, rank, device, nranks;
    cudaIpcMemHandle_t ghost[4][2];
    cudaIpcMemHandle_t ctl;        // P2PControl: epoch flags, reduction slots
    cudaIpcMemHandle_t lslab[4];   // link-slab receive buffers (halo directions, remote minus neighbour)
};
static constexpr int32_t kIpcMagic = 0x48495352;  // "HISR" (layout 2: control block + link slabs)

extern "C" int64_t dslash_ipc_blob_size(void) { return (int64_t)sizeof(IpcBlob); }

extern "C" dslash_status dslash_get_ipc_blob(dslash_t h, void* blob) {
    DeviceGuard device_guard(h);
    if (!h || !blob) return fail(h, DSLASH_ERR_ARG, "NULL argument");
    if (h->transport != DSLASH_TRANSPORT_P2P) return fail(h, DSLASH_ERR_STATE, "set DSLASH_TRANSPORT_P2P first");
    dslash_status st = alloc_lslab(h);
    if (st != DSLASH_OK) return st;
    IpcBlob b;
    memset(&b, 0, sizeof b);
    b.magic = kIpcMagic;
    b.rank = h->plan.rank;
    b.device = h->device;
    b.nranks = h->plan.nranks;
    for (int d = 2; d < 4; ++d) {
        for (int side = 0; side < 2; ++side)
            if (h->ghost[d][side]) CU(h, cudaIpcGetMemHandle(&b.ghost[d][side], h->ghost[d][side]));
        if (h->lslab[d]) CU(h, cudaIpcGetMemHandle(&b.lslab[d], h->lslab[d]));
    }
    CU(h, cudaIpcGetMemHandle(&b.ctl, h->ctl));
    memcpy(blob, &b, sizeof b);
    return DSLASH_OK;
}

// my bottom face (side 0) fills the minus neighbour's PLUS ghost, my top face (side 1) the plus
// neighbour's MINUS ghost; after consuming my ghost[d][side] I release it to the rank that filled it
static void set_peer(dslash_t h, int d, int side, char* nbr_ghost_other_side, unsigned int* nbr_flags) {
    const int other = 1 - side;
    h->peer_ghost[d][side] = nbr_ghost_other_side;
    h->peer_ready[d][side] = nbr_flags + 2 * d + other;
    h->peer_free[d][side] = nbr_flags + 8 + 2 * d + other;
}

static dslash_status ipc_open(dslash_t h, void** p, cudaIpcMemHandle_t handle) {
    CU(h, cudaIpcOpenMemHandle(p, handle, cudaIpcMemLazyEnablePeerAccess));
    h->ipc_opened.push_back(*p);
    return DSLASH_OK;
}

// Every rank's control block (reduction slots, flags); the neighbours' ghosts and the plus
// neighbours' link-slab buffers.
extern "C" dslash_status dslash_open_ipc_blobs(dslash_t h, const void* blobs) {
    DeviceGuard device_guard(h);
    if (!h || !blobs) return fail(h, DSLASH_ERR_ARG, "NULL argument");
    if (h->transport != DSLASH_TRANSPORT_P2P) return fail(h, DSLASH_ERR_STATE, "set DSLASH_TRANSPORT_P2P first");
    if (h->p2p_ready) return fail(h, DSLASH_ERR_STATE, "IPC blobs already opened");
    const dslash_plan_t& p = h->plan;
    const IpcBlob* all = static_cast<const IpcBlob*>(blobs);
    for (int r = 0; r < p.nranks; ++r)
        if (all[r].magic != kIpcMagic || all[r].rank != r || all[r].nranks != p.nranks)
            return fail(h, DSLASH_ERR_ARG, "IPC blob of rank %d is malformed or out of order", r);
    dslash_status st = alloc_lslab(h);
    if (st != DSLASH_OK) return st;
    h->peer_ctl.assign(p.nranks, nullptr);
    for (int r = 0; r < p.nranks; ++r) {
        if (r == p.rank) {
            h->peer_ctl[r] = h->ctl;
            continue;
        }
        void* cp = nullptr;
        if ((st = ipc_open(h, &cp, all[r].ctl)) != DSLASH_OK) return st;
        h->peer_ctl[r] = static_cast<P2PControl*>(cp);
    }
    for (int d = 2; d < 4; ++d) {
        if (!p.halo[d]) continue;
        for (int side = 0; side < 2; ++side) {
            const int nbr = p.nbr_rank[d][side];
            if (nbr == p.rank) {
                set_peer(h, d, side, h->ghost[d][1 - side], h->flags);
                continue;
            }
            void* gp = nullptr;
            if ((st = ipc_open(h, &gp, all[nbr].ghost[d][1 - side])) != DSLASH_OK) return st;
            set_peer(h, d, side, static_cast<char*>(gp), h->peer_ctl[nbr]->flags);
        }
        const int plus = p.nbr_rank[d][1];
        if (plus != p.rank) {
            void* lp = nullptr;
            if ((st = ipc_open(h, &lp, all[plus].lslab[d])) != DSLASH_OK) return st;
            h->peer_lslab[d] = static_cast<char*>(lp);
        }
    }
    h->p2p_ready = true;
    return DSLASH_OK;
}

// pointer setup when every neighbour is this rank (self-halo): no IPC needed
static dslash_status p2p_prepare(dslash_t h) {
    if (h->p2p_ready) return DSLASH_OK;
    const dslash_plan_t& p = h->plan;
    if (p.nranks > 1) return fail(h, DSLASH_ERR_STATE, "P2P transport: call dslash_open_ipc_blobs first");
    dslash_status st = alloc_flags(h);
    if (st != DSLASH_OK) return st;
    h->peer_ctl.assign(1, h->ctl);
    for (int d = 2; d < 4; ++d)
        if (p.halo[d])
            for (int side = 0; side < 2; ++side) set_peer(h, d, side, h->ghost[d][1 - side], h->flags);
    h->p2p_ready = true;
    return DSLASH_OK;
}

// Cross-rank gather of one double-double per rank for the solver's dot products (solver.cu
// reduce_to_slot), without NCCL: copy `mine` into slot [rank] of bank e & 1 of every rank's
// control block (copy engine; my own block too), raise red_flag[rank] = e there, and make s wait
// until every rank's flag in MY block reached e.  Bank e & 1 can be rewritten only at e + 2, and a
// rank starts e + 2 only after every rank contributed to e + 1, i.e. after every rank's stream
// finished reading e's values (the rank sum precedes its next contribution in stream order).
dslash_status hisq_p2p_gather(dslash_t h, cudaStream_t s, const double2* mine, const double2** all) {
    const dslash_plan_t& p = h->plan;
    dslash_status st = p2p_prepare(h);
    if (st != DSLASH_OK) return st;
    WriteValue32Fn wr = write_value_fn();
    WaitValue32Fn wt = wait_value_fn();
    if (!wr || !wt) return fail(h, DSLASH_ERR_UNSUPPORTED, "stream memory operations unavailable");
    const unsigned int e = ++h->red_epoch;
    const int bank = (int)(e & 1u);
    for (int r = 0; r < p.nranks; ++r)
        CU(h, cudaMemcpyAsync(&h->peer_ctl[r]->red_val[bank][p.rank], mine, sizeof(double2), cudaMemcpyDeviceToDevice, s));
    for (int r = 0; r < p.nranks; ++r)
        if (wr(s, (unsigned long long)(uintptr_t)&h->peer_ctl[r]->red_flag[p.rank], e, 0) != 0)
            return fail(h, DSLASH_ERR_CUDA, "cuStreamWriteValue32 (reduction) failed");
    for (int r = 0; r < p.nranks; ++r)
        if (wt(s, (unsigned long long)(uintptr_t)&h->ctl->red_flag[r], e, 0) != 0)
            return fail(h, DSLASH_ERR_CUDA, "cuStreamWaitValue32 (reduction) failed");
    *all = &h->ctl->red_val[bank][0];
    return DSLASH_OK;
}

// ============================================================================ halo exchange
static bool any_halo(const dslash_plan_t& p) { return p.halo[2] || p.halo[3]; }

// Face copies within this GPU (self-neighbour ghosts, the z-face pack for NCCL): up to 4 segments
// of `height` rows of `width` bytes, all in ONE kernel on the (high-priority) communication stream
// instead of cudaMemcpy2DAsync: measured on B200 the 2-D device-to-device copies of 2 x 2.36 MB
// took ~37 us beside a bandwidth-bound stencil kernel and cost it ~6.7 us per apply.  16-byte
// words when every pitch and pointer allows, else 8-byte words; 4 words per thread in flight.
// Copies to another rank's memory stay on the copy engines (cudaMemcpy2DAsync, NVLink).
struct CopySeg {
    char* dst;
    const char* src;
    size_t dpitch, spitch;
    int64_t words, rows;  // words per row, rows
};
struct CopySet {
    CopySeg seg[4];
    int n;
};

template <typename W>
__global__ void __launch_bounds__(256) face_copy_kernel(const CopySet C) {
    constexpr int U = 4;
    const CopySeg& S = C.seg[blockIdx.y];
    const int64_t n = S.words * S.rows;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i0 < n; i0 += U * stride) {
        W v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t i = i0 + u * stride;
            if (i < n) {
                const int64_t r = i / S.words, w = i - r * S.words;
                v[u] = __ldg(reinterpret_cast<const W*>(S.src + r * S.spitch) + w);  // default L2 policy: the stencil reads these lines too
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t i = i0 + u * stride;
            if (i < n) {
                const int64_t r = i / S.words, w = i - r * S.words;
                reinterpret_cast<W*>(S.dst + r * S.dpitch)[w] = v[u];
            }
        }
    }
}

static int num_sms(dslash_t h);

struct FaceCopies {
    struct Raw {
        void* dst;
        const void* src;
        size_t dpitch, spitch, width, height;
    } raw[4];
    int n = 0;
    cudaStream_t stream_of_pending = nullptr;
    // a local segment is batched; a copy into another rank's memory goes to the copy engines now
    dslash_status add(dslash_t h, void* dst, size_t dpitch, const void* src, size_t spitch, size_t width,
                      size_t height, cudaStream_t st, bool local) {
        if (!width || !height) return DSLASH_OK;
        if (!local) {
            CU(h, cudaMemcpy2DAsync(dst, dpitch, src, spitch, width, height, cudaMemcpyDeviceToDevice, st));
            return DSLASH_OK;
        }
        if (n == 4) {  // (an exchange has at most 4 local segments; flush rather than overflow)
            const dslash_status fs = flush(h, stream_of_pending);
            if (fs != DSLASH_OK) return fs;
        }
        stream_of_pending = st;
        raw[n++] = {dst, src, dpitch, spitch, width, height};
        return DSLASH_OK;
    }
    dslash_status flush(dslash_t h, cudaStream_t st) {
        if (!n) return DSLASH_OK;
        uintptr_t bits = 0;
        for (int k = 0; k < n; ++k)
            bits |= raw[k].dpitch | raw[k].spitch | raw[k].width | (uintptr_t)raw[k].dst | (uintptr_t)raw[k].src;
        const bool w16 = (bits & 15) == 0;
        const size_t ws = w16 ? 16 : 8;
        CopySet C{};
        C.n = n;
        int64_t most = 0;
        for (int k = 0; k < n; ++k) {
            C.seg[k] = {(char*)raw[k].dst, (const char*)raw[k].src, raw[k].dpitch, raw[k].spitch,
                        (int64_t)(raw[k].width / ws), (int64_t)raw[k].height};
            most = std::max<int64_t>(most, C.seg[k].words * C.seg[k].rows);
        }
        const int64_t cap = (int64_t)num_sms(h) * 8 / n;
        const dim3 grid((unsigned)std::max<int64_t>(1, std::min<int64_t>((most + 4 * 256 - 1) / (4 * 256), cap)), n);
        if (w16)
            face_copy_kernel<int4><<<grid, 256, 0, st>>>(C);
        else
            face_copy_kernel<int2><<<grid, 256, 0, st>>>(C);
        CU(h, cudaGetLastError());
        n = 0;
        return DSLASH_OK;
    }
};

// an interval of class `kind` whose start is recorded on stream s now (DSLASH_OPT_TIMING; *out =
// nullptr when timing is off); the caller records (*out)->b at its end
static dslash_status timing_begin(dslash_t h, int kind, cudaStream_t s, dslash_s::TimedLaunch** out);

// byte offset of the ghost bank that holds epoch e's faces of direction d (producer push: e & 1;
// otherwise the single bank)
static size_t bank_off(const dslash_s* h, int d, unsigned int e) { return (size_t)(e & 1u) * h->ghost_bank[d]; }

// Producer push (apply_push of epoch e = h->epoch).  Its kernels store the faces of their output
// into the neighbours' ghost bank (e + 1) & 1, which the neighbours last read at epoch e - 1 and
// release at their halo_start of epoch e: stream x (the one the pushing kernels run on) first
// waits for those releases, then the kernels run with K.push set, then x raises the neighbours'
// ready flags to e + 1 (stream memory operations: the write is fenced behind the kernels' stores).
static dslash_status push_wait_free(dslash_t h, cudaStream_t x) {
    WaitValue32Fn wt = wait_value_fn();
    for (int d = 3; d >= 2; --d)
        if (h->plan.halo[d])
            for (int side = 0; side < 2; ++side)
                if (wt(x, (unsigned long long)(uintptr_t)(h->flags + 8 + 2 * d + side), h->epoch - 1, 0) != 0)
                    return fail(h, DSLASH_ERR_CUDA, "cuStreamWaitValue32 (push free) failed");
    return DSLASH_OK;
}

static void push_params(const dslash_s* h, StencilParams& K) {
    for (int d = 2; d < 4; ++d)
        if (h->plan.halo[d]) {
            K.push_mask |= 1 << d;
            for (int side = 0; side < 2; ++side) K.push[d][side] = h->peer_ghost[d][side] + bank_off(h, d, h->epoch + 1);
        }
}

static dslash_status push_signal(dslash_t h, cudaStream_t x, const void* out, int nrhs) {
    WriteValue32Fn wr = write_value_fn();
    const unsigned int e1 = h->epoch + 1;
    for (int d = 3; d >= 2; --d)
        if (h->plan.halo[d])
            for (int side = 0; side < 2; ++side)
                if (wr(x, (unsigned long long)(uintptr_t)h->peer_ready[d][side], e1, 0) != 0)
                    return fail(h, DSLASH_ERR_CUDA, "cuStreamWriteValue32 (push ready) failed");
    h->pushed_epoch = e1;
    h->pushed_src = out;
    h->pushed_rhs = nrhs;
    return DSLASH_OK;
}

// P2P exchange of epoch e on the communication stream (copy engines + stream memory operations):
//   1. release my ghosts of epoch e-1 to the ranks that filled them (every kernel that read them
//      precedes ev_start),
//   2. wait until the ghosts my faces go to were released by their consumers (epoch e-1),
//   3. copy my bottom / top faces straight into the neighbours' ghosts (IPC-mapped),
//   4. raise their ready flags to e.
// Consumers wait for their own ready flags (halo_landed).  Every rank releases before it waits, so
// the ring of waits always resolves.
// blocked: the sources are site-blocked (dslash_apply_multi_blocked).  Every face is then a
// run of whole 16-site blocks (checked by the caller), i.e. the same byte ranges as a site-major
// layout with 3 nrhs elements per site: the copies below take es = 3 nrhs x element and one row.
static dslash_status halo_start_p2p(dslash_t h, const void* in, int nrhs, cudaStream_t s, bool blocked) {
    const dslash_plan_t& p = h->plan;
    if (nrhs > kP2PMaxRhs)
        return fail(h, DSLASH_ERR_UNSUPPORTED, "P2P transport: at most %d right-hand sides per apply", kP2PMaxRhs);
    dslash_status st = p2p_prepare(h);
    if (st != DSLASH_OK) return st;
    WriteValue32Fn wr = write_value_fn();
    WaitValue32Fn wt = wait_value_fn();
    if (!wr || !wt) return fail(h, DSLASH_ERR_UNSUPPORTED, "stream memory operations unavailable");
    const unsigned int e = h->epoch + 1;
    // producer push: the previous apply already stored this source's faces in our ghosts
    const bool pushed = h->push && h->pushed_epoch == e;
    if (pushed && (in != h->pushed_src || nrhs != h->pushed_rhs))
        return fail(h, DSLASH_ERR_STATE, "the apply after apply_push must take the pushed output as its source");
    h->epoch = e;
    h->pushed_epoch = 0;
    const size_t es = vec_elem(h) * (blocked ? 3 * nrhs : 1);
    const char* src = static_cast<const char*>(in);
    const size_t vh = (size_t)p.vh_local;
    const size_t L1 = p.local_dims[1], L2 = p.local_dims[2], L3 = p.local_dims[3];
    const size_t lxh = p.local_dims[0] / 2;
    const size_t rows = blocked ? 1 : (size_t)3 * nrhs;
    CU(h, cudaEventRecord(h->ev_start, s));
    CU(h, cudaStreamWaitEvent(h->comm, h->ev_start, 0));
    dslash_s::TimedLaunch* xt = nullptr;  // DSLASH_TIMING_EXCHANGE interval on the comm stream
    dslash_status tst = timing_begin(h, DSLASH_TIMING_EXCHANGE, h->comm, &xt);
    if (tst != DSLASH_OK) return tst;
    for (int d = 3; d >= 2; --d)
        if (p.halo[d])
            for (int side = 0; side < 2; ++side)
                if (wr(h->comm, (unsigned long long)(uintptr_t)h->peer_free[d][side], e - 1, 0) != 0)
                    return fail(h, DSLASH_ERR_CUDA, "cuStreamWriteValue32 (release) failed");
    if (pushed) {
        if (xt) CU(h, cudaEventRecord(xt->b, h->comm));  // no bytes to move: the neighbours raise our ready flags after their push
        CU(h, cudaEventRecord(h->ev_halo, h->comm));
        h->halo_pending = true;
        return DSLASH_OK;
    }
    for (int d = 3; d >= 2; --d)
        if (p.halo[d])
            for (int side = 0; side < 2; ++side)
                if (wt(h->comm, (unsigned long long)(uintptr_t)(h->flags + 8 + 2 * d + side), e - 1, 0) != 0)
                    return fail(h, DSLASH_ERR_CUDA, "cuStreamWaitValue32 (free) failed");
    // faces to another rank: copy engines (no SM; NVLink between devices); to myself: one copy kernel
    FaceCopies fc;
    if (p.halo[3]) {
        const size_t tslab = 3 * lxh * L1 * L2;
        const size_t b = bank_off(h, 3, e);
        st = fc.add(h, h->peer_ghost[3][0] + b, tslab * es, src, vh * es, tslab * es, rows, h->comm,
                    p.nbr_rank[3][0] == p.rank);
        if (st == DSLASH_OK)
            st = fc.add(h, h->peer_ghost[3][1] + b, tslab * es, src + (vh - tslab) * es, vh * es, tslab * es, rows,
                        h->comm, p.nbr_rank[3][1] == p.rank);
        if (st != DSLASH_OK) return st;
    }
    if (p.halo[2]) {
        const size_t zrow = lxh * L1;
        const size_t b = bank_off(h, 2, e);
        st = fc.add(h, h->peer_ghost[2][0] + b, 3 * zrow * es, src, L2 * zrow * es, 3 * zrow * es, rows * L3,
                    h->comm, p.nbr_rank[2][0] == p.rank);
        if (st == DSLASH_OK)
            st = fc.add(h, h->peer_ghost[2][1] + b, 3 * zrow * es, src + (L2 - 3) * zrow * es, L2 * zrow * es,
                        3 * zrow * es, rows * L3, h->comm, p.nbr_rank[2][1] == p.rank);
        if (st != DSLASH_OK) return st;
    }
    if ((st = fc.flush(h, h->comm)) != DSLASH_OK) return st;
    for (int d = 3; d >= 2; --d)
        if (p.halo[d])
            for (int side = 0; side < 2; ++side)
                if (wr(h->comm, (unsigned long long)(uintptr_t)h->peer_ready[d][side], e, 0) != 0)
                    return fail(h, DSLASH_ERR_CUDA, "cuStreamWriteValue32 (ready) failed");
    if (xt) CU(h, cudaEventRecord(xt->b, h->comm));
    CU(h, cudaEventRecord(h->ev_halo, h->comm));
    h->halo_pending = true;
    return DSLASH_OK;
}

dslash_status hisq_push_begin(dslash_t h, cudaStream_t s, FacePush* fp) {
    memset(fp, 0, sizeof *fp);
    const dslash_plan_t& p = h->plan;
    if (!h->push || !any_halo(p)) return DSLASH_OK;
    dslash_status st = p2p_prepare(h);
    if (st != DSLASH_OK) return st;
    if ((st = push_wait_free(h, s)) != DSLASH_OK) return st;
    StencilParams K{};
    push_params(h, K);
    memcpy(fp->dst, K.push, sizeof fp->dst);
    fp->mask = K.push_mask;
    fp->vh = p.vh_local;
    for (int d = 0; d < 4; ++d) fp->face_vh[d] = p.face_vh[d];
    fp->lxh = p.local_dims[0] / 2;
    fp->L1 = p.local_dims[1];
    fp->L2 = p.local_dims[2];
    fp->L3 = p.local_dims[3];
    return DSLASH_OK;
}

dslash_status hisq_push_end(dslash_t h, cudaStream_t s, const void* out) {
    if (!h->push || !any_halo(h->plan)) return DSLASH_OK;
    return push_signal(h, s, out, 1);
}

dslash_status hisq_push_discard(dslash_t h, cudaStream_t s) {
    if (!h->pushed_epoch) return DSLASH_OK;
    WriteValue32Fn wr = write_value_fn();
    const dslash_plan_t& p = h->plan;
    const unsigned int e = h->pushed_epoch;
    h->epoch = e;
    h->pushed_epoch = 0;
    CU(h, cudaEventRecord(h->ev_start, s));
    CU(h, cudaStreamWaitEvent(h->comm, h->ev_start, 0));
    for (int d = 3; d >= 2; --d)
        if (p.halo[d])
            for (int side = 0; side < 2; ++side)
                if (wr(h->comm, (unsigned long long)(uintptr_t)h->peer_free[d][side], e - 1, 0) != 0)
                    return fail(h, DSLASH_ERR_CUDA, "cuStreamWriteValue32 (release) failed");
    return DSLASH_OK;
}

// Exchange the depth-3 faces of nrhs source vectors stored back to back ([nrhs][3][vh]).
static dslash_status halo_start_impl(dslash_t h, const void* in, int nrhs, cudaStream_t s, bool blocked = false) {
    const dslash_plan_t& p = h->plan;
    if (!any_halo(p)) return DSLASH_OK;
    if (h->transport == DSLASH_TRANSPORT_P2P) return halo_start_p2p(h, in, nrhs, s, blocked);
    if (nrhs > h->ghost_rhs) {
        CU(h, cudaStreamSynchronize(h->comm));  // old ghosts may still be read by queued kernels
        CU(h, cudaDeviceSynchronize());
        dslash_status st = alloc_halo(h, nrhs);
        if (st != DSLASH_OK) return st;
    }
    // (site-blocked sources: whole 16-site blocks per face, see halo_start_p2p)
    const size_t es = vec_elem(h) * (blocked ? 3 * nrhs : 1);
    const char* src = static_cast<const char*>(in);
    const size_t vh = (size_t)p.vh_local;
    const size_t L1 = p.local_dims[1], L2 = p.local_dims[2], L3 = p.local_dims[3];
    const size_t lxh = p.local_dims[0] / 2;
    const size_t rows = blocked ? 1 : (size_t)3 * nrhs;  // (rhs, colour) rows of length vh
    CU(h, cudaEventRecord(h->ev_start, s));
    CU(h, cudaStreamWaitEvent(h->comm, h->ev_start, 0));
    dslash_s::TimedLaunch* xt = nullptr;  // DSLASH_TIMING_EXCHANGE interval on the comm stream
    dslash_status tst = timing_begin(h, DSLASH_TIMING_EXCHANGE, h->comm, &xt);
    if (tst != DSLASH_OK) return tst;
    if (h->halo_dryrun) {  // testing aid: the stream structure of the exchange without its bytes
        if (xt) CU(h, cudaEventRecord(xt->b, h->comm));
        CU(h, cudaEventRecord(h->ev_halo, h->comm));
        h->halo_pending = true;
        return DSLASH_OK;
    }
    bool nccl_work = false;
    const size_t tslab = 3 * lxh * L1 * L2;  // sites in 3 t-slices of one parity
    FaceCopies fc;                           // copies within this GPU: one kernel (flushed below)
    if (p.halo[3]) {
        if (!exch_remote(h, 3)) {
            // minus ghost <- my top slices, plus ghost <- my bottom slices (periodic self-halo)
            dslash_status st = fc.add(h, h->ghost[3][0], tslab * es, src + (vh - tslab) * es, vh * es, tslab * es,
                                      rows, h->comm, true);
            if (st == DSLASH_OK) st = fc.add(h, h->ghost[3][1], tslab * es, src, vh * es, tslab * es, rows, h->comm, true);
            if (st != DSLASH_OK) return st;
        } else {
            nccl_work = true;
        }
    }
    if (p.halo[2]) {
        // [r][c][t][z0..z0+2][y][xh] -> [r][c][t][d][y][xh]: one row of 3 z-slices per (r, c, t)
        const size_t zrow = lxh * L1;  // sites of one z-slice of one t
        const bool self = !exch_remote(h, 2);
        char* to_minus = self ? h->ghost[2][1] : h->zsend[0];  // my bottom slices
        char* to_plus = self ? h->ghost[2][0] : h->zsend[1];   // my top slices
        dslash_status st = fc.add(h, to_minus, 3 * zrow * es, src, L2 * zrow * es, 3 * zrow * es, rows * L3,
                                  h->comm, true);
        if (st == DSLASH_OK)
            st = fc.add(h, to_plus, 3 * zrow * es, src + (L2 - 3) * zrow * es, L2 * zrow * es, 3 * zrow * es,
                        rows * L3, h->comm, true);
        if (st != DSLASH_OK) return st;
        if (!self) nccl_work = true;
    }
    {
        dslash_status st = fc.flush(h, h->comm);  // the z pack precedes the sends on the comm stream
        if (st != DSLASH_OK) return st;
    }
    if (nccl_work) {
        if (!h->nccl) return fail(h, DSLASH_ERR_STATE, "halo to another rank without an NCCL communicator");
        // Per direction: sends (bottom -> minus, top -> plus) then receives (plus ghost <- plus,
        // minus ghost <- minus).  With P = 2 both neighbours are one rank and NCCL matches a pair's
        // messages in issue order: my first message (bottom) is the peer's first receive (its plus
        // ghost, since I am its plus neighbour).  Counts are bytes (ncclUint8).
        NC(h, ncclGroupStart());
        if (p.halo[3] && exch_remote(h, 3)) {
            const size_t n = tslab * es;
            for (size_t r = 0; r < rows; ++r)  // t-faces are contiguous in every (rhs, colour) row: zero copy
                NC(h, ncclSend(src + r * vh * es, n, ncclUint8, p.nbr_rank[3][0], h->nccl, h->comm));
            for (size_t r = 0; r < rows; ++r)
                NC(h, ncclSend(src + (r * vh + vh - tslab) * es, n, ncclUint8, p.nbr_rank[3][1], h->nccl, h->comm));
            for (size_t r = 0; r < rows; ++r)
                NC(h, ncclRecv(h->ghost[3][1] + r * n, n, ncclUint8, p.nbr_rank[3][1], h->nccl, h->comm));
            for (size_t r = 0; r < rows; ++r)
                NC(h, ncclRecv(h->ghost[3][0] + r * n, n, ncclUint8, p.nbr_rank[3][0], h->nccl, h->comm));
        }
        if (p.halo[2] && exch_remote(h, 2)) {
            const size_t n = rows * p.face_vh[2] * es;
            NC(h, ncclSend(h->zsend[0], n, ncclUint8, p.nbr_rank[2][0], h->nccl, h->comm));
            NC(h, ncclSend(h->zsend[1], n, ncclUint8, p.nbr_rank[2][1], h->nccl, h->comm));
            NC(h, ncclRecv(h->ghost[2][1], n, ncclUint8, p.nbr_rank[2][1], h->nccl, h->comm));
            NC(h, ncclRecv(h->ghost[2][0], n, ncclUint8, p.nbr_rank[2][0], h->nccl, h->comm));
        }
        NC(h, ncclGroupEnd());
    }
    if (xt) CU(h, cudaEventRecord(xt->b, h->comm));
    CU(h, cudaEventRecord(h->ev_halo, h->comm));
    h->halo_pending = true;
    return DSLASH_OK;
}

extern "C" dslash_status dslash_halo_start(dslash_t h, const void* in, int32_t src_parity, dslash_stream_t stream) {
    DeviceGuard device_guard(h);
    if (!h) return fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    if (!in || ((uintptr_t)in & 15)) return fail(h, DSLASH_ERR_ARG, "in is NULL or not 16-byte aligned");
    if (src_parity & ~1) return fail(h, DSLASH_ERR_ARG, "src_parity %d not in {0,1}", src_parity);
    // faces are copied in the caller's cb order; the parity only names the field
    return halo_start_impl(h, in, 1, (cudaStream_t)stream);
}

// `stream` waits until this rank's ghosts hold the current epoch's faces and its own sends are
// done (P2P: my ready flags, raised by the neighbours; NCCL / self copies: the comm event).
extern "C" dslash_status dslash_halo_wait(dslash_t h, dslash_stream_t stream) {
    DeviceGuard device_guard(h);
    if (!h) return fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    if (!h->halo_pending) return DSLASH_OK;
    if (h->transport == DSLASH_TRANSPORT_P2P) {
        WaitValue32Fn wt = wait_value_fn();
        for (int d = 3; d >= 2; --d)
            if (h->plan.halo[d])
                for (int side = 0; side < 2; ++side)
                    if (wt((cudaStream_t)stream, (unsigned long long)(uintptr_t)(h->flags + 2 * d + side), h->epoch, 0) != 0)
                        return fail(h, DSLASH_ERR_CUDA, "cuStreamWaitValue32 (ready) failed");
    }
    CU(h, cudaStreamWaitEvent((cudaStream_t)stream, h->ev_halo, 0));
    h->halo_pending = false;
    return DSLASH_OK;
}

// ============================================================================ launches
static void fill_boxes(StencilParams& K, const dslash_box_t* boxes, int n) {
    K.nbox = n;
    K.box_start[0] = 0;
    for (int b = 0; b < n; ++b) {
        for (int d = 0; d < 4; ++d) {
            K.box[b].lo[d] = boxes[b].lo[d];
            K.box[b].n[d] = boxes[b].hi[d] - boxes[b].lo[d];
        }
        K.div_xh[b].init((uint32_t)(K.box[b].n[0] / 2));
        K.div_y[b].init((uint32_t)K.box[b].n[1]);
        K.div_z[b].init((uint32_t)K.box[b].n[2]);
        K.box_start[b + 1] = K.box_start[b] + (int64_t)(K.box[b].n[0] / 2) * K.box[b].n[1] * K.box[b].n[2] * K.box[b].n[3];
    }
    for (int b = n; b < kMaxBoxes; ++b) K.box_start[b + 1] = K.box_start[n];
}

static StencilFn pick_vblk_kernel(int precision, int recon, bool ghost, int lanes, int nrhs) {
    if (recon == 9)
        return precision == DSLASH_F32     ? pick_f32_r9_vblk(ghost, lanes, nrhs)
               : precision == DSLASH_MIXED ? pick_mixed_r9_vblk(ghost, lanes, nrhs)
                                           : pick_f64_r9_vblk(ghost, lanes, nrhs);
    const bool r12 = recon == 12;
    switch (precision) {
        case DSLASH_F32: return r12 ? pick_f32_r12_vblk(ghost, lanes, nrhs) : pick_f32_r18_vblk(ghost, lanes, nrhs);
        case DSLASH_MIXED:
            return r12 ? pick_mixed_r12_vblk(ghost, lanes, nrhs) : pick_mixed_r18_vblk(ghost, lanes, nrhs);
        default: return r12 ? pick_f64_r12_vblk(ghost, lanes, nrhs) : pick_f64_r18_vblk(ghost, lanes, nrhs);
    }
}

template <bool GHOST>
static StencilFn pick_kernel(int precision, int recon, int lanes, int minb, int nrhs) {
    const bool r12 = recon == 12;
    if (recon == 9)
        return precision == DSLASH_F32     ? pick_f32_r9(GHOST, lanes, minb, nrhs)
               : precision == DSLASH_MIXED ? pick_mixed_r9(GHOST, lanes, minb, nrhs)
                                           : pick_f64_r9(GHOST, lanes, minb, nrhs);
    switch (precision) {
        case DSLASH_F32: return r12 ? pick_f32_r12(GHOST, lanes, minb, nrhs) : pick_f32_r18(GHOST, lanes, minb, nrhs);
        case DSLASH_MIXED: return r12 ? pick_mixed_r12(GHOST, lanes, minb, nrhs) : pick_mixed_r18(GHOST, lanes, minb, nrhs);
        default: return r12 ? pick_f64_r12(GHOST, lanes, minb, nrhs) : pick_f64_r18(GHOST, lanes, minb, nrhs);
    }
}

// defaults chosen by measurement on B200 (tools/sweep.py; profiles/README.md): at 32^4 and 48^4
// every mapping is best at <= 128 registers (min 2 blocks of 256), LANES 1/2 at 64-128 threads
// (4 / 8 right-hand sides: 128 / 256-thread blocks, 229.0 vs 231.7 us and 382-389 vs 390-400 us at
// 64; profiles/r02/mrhs/, profiles/r02/misc/)
static constexpr int kDefaultBlock = 64, kDefaultBlockRhs4 = 128, kDefaultBlockRhs8 = 256, kDefaultMinBlocks = 2;

static StencilFn pick_stage_kernel(int precision, int recon, bool ghost, int lanes, int nrhs) {
    const bool r12 = recon == 12;
    if (recon == 9)
        return precision == DSLASH_F32     ? pick_f32_r9_stage(ghost, lanes, nrhs)
               : precision == DSLASH_MIXED ? pick_mixed_r9_stage(ghost, lanes, nrhs)
                                           : pick_f64_r9_stage(ghost, lanes, nrhs);
    switch (precision) {
        case DSLASH_F32:
            return r12 ? pick_f32_r12_stage(ghost, lanes, nrhs) : pick_f32_r18_stage(ghost, lanes, nrhs);
        case DSLASH_MIXED:
            return r12 ? pick_mixed_r12_stage(ghost, lanes, nrhs) : pick_mixed_r18_stage(ghost, lanes, nrhs);
        default: return r12 ? pick_f64_r12_stage(ghost, lanes, nrhs) : pick_f64_r18_stage(ghost, lanes, nrhs);
    }
}

// rows per tile of the neighbour-staged kernel: the largest divisor TY of Ly with
// lxh * TY * threads_per_site <= 256 (0: an x-row alone exceeds a block)
static int stage_rows(const dslash_s* h, int threads_per_site) {
    const int lxh = h->plan.local_dims[0] / 2, Ly = h->plan.local_dims[1];
    for (int ty = Ly; ty >= 1; --ty)
        if (Ly % ty == 0 && lxh * ty * threads_per_site <= 256) return ty;
    return 0;
}

// events around one timed launch (DSLASH_OPT_TIMING); *out = NULL when timing is off
static dslash_status timing_begin(dslash_t h, int kind, cudaStream_t s, dslash_s::TimedLaunch** out) {
    *out = nullptr;
    if (!h->timing) return DSLASH_OK;
    if (h->tused == h->tpool.size()) {
        dslash_s::TimedLaunch t{};
        CU(h, cudaEventCreate(&t.a));
        CU(h, cudaEventCreate(&t.b));
        h->tpool.push_back(t);
    }
    dslash_s::TimedLaunch* tl = &h->tpool[h->tused++];
    tl->kind = kind;
    CU(h, cudaEventRecord(tl->a, s));
    *out = tl;
    return DSLASH_OK;
}

// launch with programmatic stream serialization (the kernels wait with griddepcontrol.wait before
// touching psi or chi, stencil.cuh) or as an ordinary launch
static cudaError_t launch_pdl(bool pdl, StencilFn fn, const StencilParams& K, unsigned grid, int bs, size_t smem,
                              cudaStream_t s) {
    // HISQ_L1_CARVEOUT=<percent>: shared-memory carveout preference of the stencil kernels
    // (0 = largest L1), set once per kernel; a measurement aid
    static const char* cv = getenv("HISQ_L1_CARVEOUT");
    if (cv) {
        static std::vector<StencilFn> done;
        bool seen = false;
        for (StencilFn f : done) seen = seen || f == fn;
        if (!seen) {
            done.push_back(fn);
            cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, atoi(cv));
        }
    }
    if (!pdl) {
        fn<<<grid, bs, smem, s>>>(K);
        return cudaGetLastError();
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(bs);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, fn, K);
}

// the neighbour-staged kernel over the boxes of K: one block per tile of TY full x-rows
static dslash_status launch_stage(dslash_t h, StencilParams K, bool ghost, int kind, cudaStream_t s, int nrhs,
                                  int lanes) {
    const int64_t sites = K.box_start[K.nbox];
    // cp.async.bulk copies whole x-rows: sizes and shared-memory offsets must be 16-byte
    // multiples (checked here, not only in set_option: dslash_cg_mixed runs an F64 handle's
    // staged kernels as F32 ones)
    if ((K.lxh * vec_elem(h)) % 16)
        return fail(h, DSLASH_ERR_UNSUPPORTED, "staged kernel: an x-row of %d sites x %zu B is not a 16-byte multiple",
                    K.lxh, vec_elem(h));
    const int rhsl = nrhs == 8 ? 2 : 1;
    const int ty = stage_rows(h, lanes * rhsl);
    if (!ty)
        return fail(h, DSLASH_ERR_UNSUPPORTED, "staged kernel: an x-row of %d sites x %d threads exceeds a block",
                    K.lxh, lanes * rhsl);
    K.stage_ty = ty;
    const int64_t tile = (int64_t)K.lxh * ty;  // every box holds whole tiles (full x and y extents)
    const unsigned grid = (unsigned)(sites / tile);
    const int bs = (int)(tile * lanes * rhsl);
    const size_t smem = (size_t)nrhs * 3 * (ty + 6) * K.lxh * vec_elem(h);
    StencilFn fn = pick_stage_kernel(h->precision, h->recon, ghost, lanes, nrhs);
    static std::vector<std::pair<StencilFn, size_t>> smem_set;  // opt-in above 48 KB, once per size
    if (smem > 48 * 1024) {
        bool done = false;
        for (auto& e : smem_set)
            if (e.first == fn && e.second >= smem) done = true;
        if (!done) {
            CU(h, cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            smem_set.push_back({fn, smem});
        }
    }
    dslash_s::TimedLaunch* tl = nullptr;
    dslash_status st = timing_begin(h, kind, s, &tl);
    if (st != DSLASH_OK) return st;
    CU(h, launch_pdl(h->pdl, fn, K, grid, bs, smem, s));
    if (tl) CU(h, cudaEventRecord(tl->b, s));
    return DSLASH_OK;
}

// one launch of the stencil over the boxes of K for nrhs (1, 2, 4 or 8) right-hand sides
static int num_sms(dslash_t h) {
    static int n = 0;
    if (!n && cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, h->device) != cudaSuccess) n = 148;
    return n;
}

static dslash_status launch(dslash_t h, const StencilParams& K, bool ghost, int kind, cudaStream_t s, int nrhs) {
    const int64_t sites = K.box_start[K.nbox];
    if (sites == 0) return DSLASH_OK;
    const int lanes = lanes_of(h->kernel);
    if (h->stage && !K.vblk) return launch_stage(h, K, ghost, kind, s, nrhs, lanes);
    // recon-9 on the site kernel (its default): 256 / 128 / 64 threads for fp64 / mixed / fp32
    // (profiles/r02/recon9_blocks/: 150.6 vs 152.7 us, 86.9 vs 88.0 us, 75.9 vs 77.3 us)
    const int r9_block = h->precision == DSLASH_F64 ? 256 : h->precision == DSLASH_MIXED ? 128 : 64;
    const int bs = h->block                        ? h->block
                   : nrhs == 8                     ? kDefaultBlockRhs8
                   : nrhs == 4                     ? kDefaultBlockRhs4
                   : (h->recon == 9 && lanes == 1) ? r9_block
                                                   : kDefaultBlock;
    const int minb = h->min_blocks ? h->min_blocks : kDefaultMinBlocks;
    // right-hand sides are register-blocked per thread; 8 of them use 2 thread groups of 4, except
    // interior site-blocked launches without recon-9 (one group of 8: kernels_inst.cuh pick_vblk_n)
    const int vblk_groups8 = (h->recon == 9 || ghost) ? 2 : 1;
    const int64_t threads = sites * lanes * (nrhs == 8 ? (K.vblk ? vblk_groups8 : 2) : 1);
    const unsigned grid = (unsigned)((threads + bs - 1) / bs);
    dslash_s::TimedLaunch* tl = nullptr;
    dslash_status st = timing_begin(h, kind, s, &tl);
    if (st != DSLASH_OK) return st;
    StencilFn fn = K.vblk  ? pick_vblk_kernel(h->precision, h->recon, ghost, lanes, nrhs)
                   : ghost ? pick_kernel<true>(h->precision, h->recon, lanes, minb, nrhs)
                           : pick_kernel<false>(h->precision, h->recon, lanes, minb, nrhs);
    // programmatic dependent launch: may start while the previous kernel on `s` drains
    CU(h, launch_pdl(h->pdl, fn, K, grid, bs, 0, s));
    if (tl) CU(h, cudaEventRecord(tl->b, s));
    return DSLASH_OK;
}

// launch over `boxes` for all nrhs right-hand sides, in chunks of 8, 4, 2, 1
static dslash_status launch_rhs(dslash_t h, StencilParams K, const dslash_box_t* boxes, int nbox, bool ghost,
                                int kind, cudaStream_t s, int nrhs) {
    fill_boxes(K, boxes, nbox);
    const size_t es = vec_elem(h);
    const char* in0 = static_cast<const char*>(K.in);
    char* out0 = static_cast<char*>(K.out);
    const void* g0[4][2];
    memcpy(g0, K.ghost, sizeof g0);
    void* p0[4][2];
    memcpy(p0, K.push, sizeof p0);
    for (int r0 = 0; r0 < nrhs;) {
        const int left = nrhs - r0;
        int nr = left >= 8 ? 8 : left >= 4 ? 4 : left >= 2 ? 2 : 1;
        // planar: the chunk's first vector; site-blocked: its first rows inside every 16-site block
        const size_t roff = (size_t)r0 * 3 * (K.vblk ? kVBlk : K.vh) * es;
        K.in = in0 + roff;
        K.out = out0 + roff;
        for (int d = 0; d < 4; ++d)
            for (int side = 0; side < 2; ++side) {
                K.ghost[d][side] = g0[d][side] ? static_cast<const char*>(g0[d][side]) +
                                                     (size_t)r0 * 3 * (K.vblk ? kVBlk : K.face_vh[d]) * es
                                               : nullptr;
                K.push[d][side] = p0[d][side] ? static_cast<char*>(p0[d][side]) + (size_t)r0 * 3 * K.face_vh[d] * es
                                              : nullptr;
            }
        dslash_status st = launch(h, K, ghost, kind, s, nr);
        if (st != DSLASH_OK) return st;
        r0 += nr;
    }
    return DSLASH_OK;
}

static dslash_status check_vectors(dslash_t h, const void* out, const void* in, int nrhs) {
    if (!out || !in) return fail(h, DSLASH_ERR_ARG, "NULL vector pointer");
    if (((uintptr_t)out & 15) || ((uintptr_t)in & 15)) return fail(h, DSLASH_ERR_ARG, "vectors must be 16-byte aligned");
    const uintptr_t n = (uintptr_t)nrhs * 3 * h->plan.vh_local * vec_elem(h);
    const uintptr_t a = (uintptr_t)out, b = (uintptr_t)in;
    if (a < b + n && b < a + n) return fail(h, DSLASH_ERR_ARG, "in and out overlap");
    return DSLASH_OK;
}

static dslash_status apply_impl(dslash_t h, void* out, const void* in, int32_t parity, int32_t nrhs,
                                dslash_stream_t stream, bool push_out = false, bool blocked = false);

dslash_status hisq_apply(dslash_t h, void* out, const void* in, int32_t parity, int32_t nrhs, cudaStream_t s,
                         bool push) {
    return apply_impl(h, out, in, parity, nrhs, (dslash_stream_t)s, push);
}

static dslash_status apply_impl(dslash_t h, void* out, const void* in, int32_t parity, int32_t nrhs,
                                dslash_stream_t stream, bool push_out, bool blocked) {
    DeviceGuard device_guard(h);
    if (!h) return fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    if (parity & ~1) return fail(h, DSLASH_ERR_ARG, "parity %d not in {0,1}", parity);
    if (nrhs < 1) return fail(h, DSLASH_ERR_ARG, "nrhs %d < 1", nrhs);
    if (h->parity_mask != DSLASH_BOTH && h->parity_mask != parity)
        return fail(h, DSLASH_ERR_ARG, "parity %d not prepared (parity_mask %d)", parity, h->parity_mask);
    if (!h->loaded) return fail(h, DSLASH_ERR_STATE, "apply before load_links");
    dslash_status st = check_vectors(h, out, in, nrhs);
    if (st != DSLASH_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    const dslash_plan_t& p = h->plan;
    StencilParams K{};
    K.links = h->links[parity];
    K.in = in;
    K.out = out;
    K.vh = p.vh_local;
    K.lxh = p.local_dims[0] / 2;
    K.parity = parity;
    K.long_inv_scale = h->long_inv_scale;
    K.long_scale = h->long_scale;
    for (int d = 0; d < 4; ++d) {
        K.L[d] = p.local_dims[d];
        K.face_vh[d] = p.face_vh[d];
        if (p.halo[d]) K.halo_mask |= 1 << d;
    }
    // producer push: only with a halo (without one the next apply needs no faces)
    push_out = push_out && any_halo(p);
    if (push_out && !h->push) return fail(h, DSLASH_ERR_STATE, "apply_push needs DSLASH_OPT_PUSH");
    if (blocked) {  // site-blocked vectors (dslash_apply_multi_blocked)
        // every face exchanged must be a run of whole 16-site blocks: the t face (3 t-slices), and
        // per t-slice the 3 bottom / top z-slices, with their offsets
        const int64_t zrow = (int64_t)K.lxh * K.L[1];
        const bool ok = p.vh_local % kVBlk == 0 && (!p.halo[3] || (3 * zrow * K.L[2]) % kVBlk == 0) &&
                        (!p.halo[2] || ((3 * zrow) % kVBlk == 0 && (zrow * K.L[2]) % kVBlk == 0));
        if (!ok)
            return fail(h, DSLASH_ERR_UNSUPPORTED,
                        "site-blocked layout: Vh_local and every exchanged face must be whole blocks of %d sites", kVBlk);
        if (any_halo(p) && (push_out || h->overlap == DSLASH_OVERLAP_DIRS))
            return fail(h, DSLASH_ERR_UNSUPPORTED,
                        "site-blocked layout: no producer push and no split-by-direction overlap");
        K.vblk = (int64_t)nrhs * 3 * kVBlk;
    }
    if (!any_halo(p)) return launch_rhs(h, K, p.interior, p.n_interior, false, DSLASH_TIMING_INTERIOR, s, nrhs);
    if ((st = halo_start_impl(h, in, nrhs, s, blocked)) != DSLASH_OK) return st;
    for (int d = 0; d < 4; ++d) {  // after halo_start: the ghosts may have been (re)allocated
        K.ghost[d][0] = h->ghost[d][0] ? h->ghost[d][0] + bank_off(h, d, h->epoch) : nullptr;
        K.ghost[d][1] = h->ghost[d][1] ? h->ghost[d][1] + bank_off(h, d, h->epoch) : nullptr;
    }
    // the interior launches never push (no interior site lies within 3 slices of a face)
    StencilParams Kp = K;
    if (push_out) push_params(h, Kp);
    if (h->overlap == DSLASH_OVERLAP_DIRS) {
        // split by direction: the local pass runs over EVERY site while the faces are in flight,
        // skipping the hops into ghost faces; once they landed, the ghost pass adds exactly those
        // hops to the boundary sites' partial sums (QUDA-style interior / exterior kernels).  Both
        // on the caller's stream; the bench reports their span.
        size_t span = (size_t)-1;
        if (h->timing) {
            dslash_s::TimedLaunch* tl = nullptr;
            if ((st = timing_begin(h, DSLASH_TIMING_SPAN, s, &tl)) != DSLASH_OK) return st;
            span = (size_t)(tl - h->tpool.data());
        }
        K.halo_pass = kPassLocal;
        if (p.n_interior + p.n_boundary > kMaxBoxes) {
            st = launch_rhs(h, K, p.interior, p.n_interior, true, DSLASH_TIMING_INTERIOR, s, nrhs);
            if (st == DSLASH_OK)
                st = launch_rhs(h, K, p.boundary, p.n_boundary, true, DSLASH_TIMING_INTERIOR, s, nrhs);
        } else {
            dslash_box_t all[kMaxBoxes];
            int n = 0;
            for (int i = 0; i < p.n_interior; ++i) all[n++] = p.interior[i];
            for (int i = 0; i < p.n_boundary; ++i) all[n++] = p.boundary[i];
            st = launch_rhs(h, K, all, n, true, DSLASH_TIMING_INTERIOR, s, nrhs);
        }
        if (st != DSLASH_OK) return st;
        if ((st = dslash_halo_wait(h, stream)) != DSLASH_OK) return st;
        if (push_out && (st = push_wait_free(h, s)) != DSLASH_OK) return st;
        Kp.halo_pass = kPassGhost;
        if ((st = launch_rhs(h, Kp, p.boundary, p.n_boundary, true, DSLASH_TIMING_BOUNDARY, s, nrhs)) != DSLASH_OK)
            return st;
        if (push_out && (st = push_signal(h, s, out, nrhs)) != DSLASH_OK) return st;
        if (span != (size_t)-1) CU(h, cudaEventRecord(h->tpool[span].b, s));
        return DSLASH_OK;
    }
    // without interior sites (e.g. 48^4 on 8 GPUs, local Lt = 6) nothing can overlap the exchange:
    // one launch on the caller's stream after it, no boundary stream and join (measured equal,
    // 153.7 vs 153.8 us per apply at 48^3 x 6 with a t self-halo)
    if (h->overlap == DSLASH_OVERLAP_SITES && p.interior_sites > 0) {
        // interior on the caller's stream; boundary on the exchange stream as soon as the halo
        // lands, so it fills the SMs the interior kernel's tail leaves idle; then the caller's
        // stream joins (the two kernels write disjoint sites of out)
        // span of the two overlapping kernels (DSLASH_TIMING_SPAN): interior start -> join
        // (an index, not a pointer: the launches below may grow tpool)
        size_t span = (size_t)-1;
        if (h->timing) {
            if (h->tused == h->tpool.size()) {
                dslash_s::TimedLaunch t{};
                CU(h, cudaEventCreate(&t.a));
                CU(h, cudaEventCreate(&t.b));
                h->tpool.push_back(t);
            }
            span = h->tused++;
            h->tpool[span].kind = DSLASH_TIMING_SPAN;
            CU(h, cudaEventRecord(h->tpool[span].a, s));
        }
        // the boundary kernel is queued on the exchange's own (high-priority) stream right behind
        // the exchange: no cross-stream wait between the faces and the kernel that reads them
        // (round 3, profiles/r03/halo/: t 185.2 -> 182.9 us, t + z 186.7 -> 185.0 us per apply
        // against 178.9 us without a halo, vs a separate boundary stream)
        cudaStream_t bs = h->comm;
        st = launch_rhs(h, K, p.interior, p.n_interior, false, DSLASH_TIMING_INTERIOR, s, nrhs);
        if (st != DSLASH_OK) return st;
        if ((st = dslash_halo_wait(h, (dslash_stream_t)bs)) != DSLASH_OK) return st;
        if (push_out && (st = push_wait_free(h, bs)) != DSLASH_OK) return st;
        st = launch_rhs(h, Kp, p.boundary, p.n_boundary, true, DSLASH_TIMING_BOUNDARY, bs, nrhs);
        if (st != DSLASH_OK) return st;
        if (push_out && (st = push_signal(h, bs, out, nrhs)) != DSLASH_OK) return st;
        CU(h, cudaEventRecord(h->ev_bdone, bs));
        CU(h, cudaStreamWaitEvent(s, h->ev_bdone, 0));
        if (span != (size_t)-1) CU(h, cudaEventRecord(h->tpool[span].b, s));
        return DSLASH_OK;
    }
    if ((st = dslash_halo_wait(h, stream)) != DSLASH_OK) return st;
    if (push_out && (st = push_wait_free(h, s)) != DSLASH_OK) return st;
    if (p.n_interior + p.n_boundary > kMaxBoxes) {
        // 5 boxes (t and z halo): launch the interior part first, then the boundary boxes
        st = launch_rhs(h, K, p.interior, p.n_interior, true, DSLASH_TIMING_INTERIOR, s, nrhs);
        if (st == DSLASH_OK) st = launch_rhs(h, Kp, p.boundary, p.n_boundary, true, DSLASH_TIMING_BOUNDARY, s, nrhs);
    } else {
        dslash_box_t all[kMaxBoxes];
        int n = 0;
        for (int i = 0; i < p.n_interior; ++i) all[n++] = p.interior[i];
        for (int i = 0; i < p.n_boundary; ++i) all[n++] = p.boundary[i];
        st = launch_rhs(h, Kp, all, n, true, DSLASH_TIMING_ALL, s, nrhs);
    }
    if (st == DSLASH_OK && push_out) st = push_signal(h, s, out, nrhs);
    return st;
}

extern "C" dslash_status dslash_apply(dslash_t h, void* out, const void* in, int32_t parity, dslash_stream_t stream) {
    return apply_impl(h, out, in, parity, 1, stream);
}

extern "C" dslash_status dslash_apply_push(dslash_t h, void* out, const void* in, int32_t parity,
                                           dslash_stream_t stream) {
    return apply_impl(h, out, in, parity, 1, stream, true);
}

extern "C" dslash_status dslash_apply_multi_blocked(dslash_t h, int32_t nrhs, void* out, const void* in,
                                                    int32_t parity, dslash_stream_t stream) {
    return apply_impl(h, out, in, parity, nrhs, stream, false, true);
}

dslash_status hisq_apply_blocked(dslash_t h, void* out, const void* in, int32_t parity, int32_t nrhs, cudaStream_t s) {
    return apply_impl(h, out, in, parity, nrhs, (dslash_stream_t)s, false, true);
}

// planar [rows][vh] <-> site-blocked [vh / 16][rows][16] (rows = 3 nrhs), one element per thread in
// the blocked order, so both sides move runs of 16 consecutive elements
template <typename T>
__global__ void vblk_convert_kernel(T* __restrict__ dst, const T* __restrict__ src, int64_t vh, int rows,
                                    bool to_blocked) {
    const int64_t n = vh * rows, blk = (int64_t)rows * kVBlk;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t b = i / blk, rem = i - b * blk;
        const int64_t planar = (rem / kVBlk) * vh + b * kVBlk + rem % kVBlk;
        if (to_blocked)
            dst[i] = src[planar];
        else
            dst[planar] = src[i];
    }
}

static dslash_status vblk_convert(dslash_t h, int32_t nrhs, void* dst, const void* src, dslash_stream_t stream,
                                  bool to_blocked) {
    DeviceGuard device_guard(h);
    if (!h) return fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    if (nrhs < 1) return fail(h, DSLASH_ERR_ARG, "nrhs %d < 1", nrhs);
    dslash_status st = check_vectors(h, dst, src, nrhs);
    if (st != DSLASH_OK) return st;
    const int64_t vh = h->plan.vh_local;
    if (vh % kVBlk)
        return fail(h, DSLASH_ERR_UNSUPPORTED, "site-blocked layout: Vh_local %lld is not a multiple of %d",
                    (long long)vh, kVBlk);
    const int rows = 3 * nrhs;
    const unsigned grid = (unsigned)std::min<int64_t>((vh * rows + 255) / 256, (int64_t)num_sms(h) * 8);
    cudaStream_t s = (cudaStream_t)stream;
    if (vec_elem(h) == 16)
        vblk_convert_kernel<double2><<<grid, 256, 0, s>>>(static_cast<double2*>(dst), static_cast<const double2*>(src),
                                                          vh, rows, to_blocked);
    else
        vblk_convert_kernel<float2><<<grid, 256, 0, s>>>(static_cast<float2*>(dst), static_cast<const float2*>(src), vh,
                                                         rows, to_blocked);
    CU(h, cudaGetLastError());
    return DSLASH_OK;
}

extern "C" dslash_status dslash_vectors_to_blocked(dslash_t h, int32_t nrhs, void* blocked, const void* planar,
                                                   dslash_stream_t stream) {
    return vblk_convert(h, nrhs, blocked, planar, stream, true);
}

extern "C" dslash_status dslash_vectors_from_blocked(dslash_t h, int32_t nrhs, void* planar, const void* blocked,
                                                     dslash_stream_t stream) {
    return vblk_convert(h, nrhs, planar, blocked, stream, false);
}

extern "C" dslash_status dslash_apply_multi(dslash_t h, int32_t nrhs, void* out, const void* in, int32_t parity,
                                            dslash_stream_t stream) {
    return apply_impl(h, out, in, parity, nrhs, stream);
}

extern "C" dslash_status dslash_apply_host(dslash_t h, void* out_host, const void* in_host, int32_t parity,
                                           dslash_stream_t stream) {
    DeviceGuard device_guard(h);
    if (!h) return fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    if (!out_host || !in_host) return fail(h, DSLASH_ERR_ARG, "NULL host buffer");
    const size_t bytes = 3 * (size_t)h->plan.vh_local * vec_elem(h);
    if (!h->stage_in) CU(h, cudaMalloc(&h->stage_in, bytes));
    if (!h->stage_out) CU(h, cudaMalloc(&h->stage_out, bytes));
    cudaStream_t s = (cudaStream_t)stream;
    CU(h, cudaMemcpyAsync(h->stage_in, in_host, bytes, cudaMemcpyHostToDevice, s));
    dslash_status st = dslash_apply(h, h->stage_out, h->stage_in, parity, stream);
    if (st != DSLASH_OK) return st;
    CU(h, cudaMemcpyAsync(out_host, h->stage_out, bytes, cudaMemcpyDeviceToHost, s));
    return DSLASH_OK;
}

extern "C" dslash_status dslash_apply_host_batch(dslash_t h, int32_t n, void* const* out_host,
                                                 const void* const* in_host, int32_t parity,
                                                 dslash_stream_t stream) {
    DeviceGuard device_guard(h);
    if (!h) return fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    if (n < 0 || (n > 0 && (!out_host || !in_host))) return fail(h, DSLASH_ERR_ARG, "bad batch arguments");
    if (!h->loaded) return fail(h, DSLASH_ERR_STATE, "apply before load_links");
    for (int32_t i = 0; i < n; ++i)
        if (!out_host[i] || !in_host[i]) return fail(h, DSLASH_ERR_ARG, "NULL host buffer in batch entry %d", i);
    if (n == 0) return DSLASH_OK;
    const int S = dslash_s::kSlots;
    const size_t bytes = 3 * (size_t)h->plan.vh_local * vec_elem(h);
    if (!h->h2d) {
        CU(h, cudaStreamCreateWithFlags(&h->h2d, cudaStreamNonBlocking));
        CU(h, cudaStreamCreateWithFlags(&h->d2h, cudaStreamNonBlocking));
        CU(h, cudaEventCreateWithFlags(&h->ev_batch, cudaEventDisableTiming));
        for (int k = 0; k < S; ++k) {
            CU(h, cudaMalloc(&h->slot_in[k], bytes));
            CU(h, cudaMalloc(&h->slot_out[k], bytes));
            CU(h, cudaEventCreateWithFlags(&h->ev_in_ready[k], cudaEventDisableTiming));
            CU(h, cudaEventCreateWithFlags(&h->ev_in_free[k], cudaEventDisableTiming));
            CU(h, cudaEventCreateWithFlags(&h->ev_out_ready[k], cudaEventDisableTiming));
            CU(h, cudaEventCreateWithFlags(&h->ev_out_free[k], cudaEventDisableTiming));
            // slots start free
            CU(h, cudaEventRecord(h->ev_in_free[k], h->h2d));
            CU(h, cudaEventRecord(h->ev_out_free[k], h->d2h));
        }
    }
    cudaStream_t s = (cudaStream_t)stream;
    CU(h, cudaEventRecord(h->ev_batch, s));
    CU(h, cudaStreamWaitEvent(h->h2d, h->ev_batch, 0));
    for (int32_t i = 0; i < n; ++i) {
        const int k = i % S;
        // H2D into slot k once the apply that last read it has finished
        CU(h, cudaStreamWaitEvent(h->h2d, h->ev_in_free[k], 0));
        CU(h, cudaMemcpyAsync(h->slot_in[k], in_host[i], bytes, cudaMemcpyHostToDevice, h->h2d));
        CU(h, cudaEventRecord(h->ev_in_ready[k], h->h2d));
        // apply on the caller's stream once the input landed and the output slot was drained
        CU(h, cudaStreamWaitEvent(s, h->ev_in_ready[k], 0));
        CU(h, cudaStreamWaitEvent(s, h->ev_out_free[k], 0));
        dslash_status st = dslash_apply(h, h->slot_out[k], h->slot_in[k], parity, stream);
        if (st != DSLASH_OK) return st;
        CU(h, cudaEventRecord(h->ev_in_free[k], s));
        CU(h, cudaEventRecord(h->ev_out_ready[k], s));
        // D2H of the result
        CU(h, cudaStreamWaitEvent(h->d2h, h->ev_out_ready[k], 0));
        CU(h, cudaMemcpyAsync(out_host[i], h->slot_out[k], bytes, cudaMemcpyDeviceToHost, h->d2h));
        CU(h, cudaEventRecord(h->ev_out_free[k], h->d2h));
    }
    CU(h, cudaEventRecord(h->ev_batch, h->d2h));
    CU(h, cudaStreamWaitEvent(s, h->ev_batch, 0));
    return DSLASH_OK;
}

// ============================================================================ misc
extern "C" dslash_status dslash_sync(dslash_t h) {
    DeviceGuard device_guard(h);
    if (!h) return fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    CU(h, cudaStreamSynchronize(h->comm));
    CU(h, cudaDeviceSynchronize());
    if (h->nccl) {
        ncclResult_t async_err;
        NC(h, ncclCommGetAsyncError(h->nccl, &async_err));
        if (async_err != ncclSuccess)
            return fail(h, DSLASH_ERR_NCCL, "NCCL async error: %s", ncclGetErrorString(async_err));
    }
    return h->err;
}

extern "C" dslash_status dslash_kernel_timing(dslash_t h, int32_t which, double* total_ms, int64_t* launches) {
    DeviceGuard device_guard(h);
    if (!h) return fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    if (!total_ms || !launches) return fail(h, DSLASH_ERR_ARG, "NULL output");
    double tot = 0.0;
    int64_t n = 0;
    for (size_t i = 0; i < h->tused; ++i) {
        const auto& t = h->tpool[i];
        // ALL = every kernel launch (spans excluded: they cover launches already counted; exchanges
        // are not kernels of this library)
        if (which == DSLASH_TIMING_ALL ? (t.kind == DSLASH_TIMING_SPAN || t.kind == DSLASH_TIMING_EXCHANGE)
                                       : t.kind != which)
            continue;
        CU(h, cudaEventSynchronize(t.b));
        float ms = 0.f;
        CU(h, cudaEventElapsedTime(&ms, t.a, t.b));
        tot += ms;
        ++n;
    }
    *total_ms = tot;
    *launches = n;
    return DSLASH_OK;
}

extern "C" dslash_status dslash_timeline(dslash_t h, int64_t max_entries, int32_t* kinds, double* start_ms,
                                         double* end_ms, int64_t* n) {
    DeviceGuard device_guard(h);
    if (!h) return fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    if (!n || (max_entries > 0 && (!kinds || !start_ms || !end_ms))) return fail(h, DSLASH_ERR_ARG, "NULL output");
    *n = (int64_t)h->tused;
    for (size_t i = 0; i < h->tused && (int64_t)i < max_entries; ++i) {
        const auto& t = h->tpool[i];
        CU(h, cudaEventSynchronize(t.b));
        float a = 0.f, b = 0.f;
        CU(h, cudaEventElapsedTime(&a, h->tpool[0].a, t.a));
        CU(h, cudaEventElapsedTime(&b, h->tpool[0].a, t.b));
        kinds[i] = t.kind;
        start_ms[i] = a;
        end_ms[i] = b;
    }
    return DSLASH_OK;
}

extern "C" dslash_status dslash_kernel_timing_reset(dslash_t h) {
    DeviceGuard device_guard(h);
    if (!h) return fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    if (h->tused) CU(h, cudaEventSynchronize(h->tpool[h->tused - 1].b));
    h->tused = 0;
    return DSLASH_OK;
}

extern "C" dslash_status dslash_get_plan(dslash_t h, dslash_plan_t* plan) {
    if (!h || !plan) return fail(h, DSLASH_ERR_ARG, "NULL argument");
    *plan = h->plan;
    return DSLASH_OK;
}

extern "C" int64_t dslash_local_half_volume(dslash_t h) { return h ? h->plan.vh_local : -1; }

extern "C" dslash_status dslash_destroy(dslash_t h) {
    DeviceGuard device_guard(h);
    if (!h) return DSLASH_OK;
    if (h->comm) cudaStreamSynchronize(h->comm);
    cudaDeviceSynchronize();
    free_links(h);
    free_halo(h);
    if (h->stage_in) cudaFree(h->stage_in);
    if (h->stage_out) cudaFree(h->stage_out);
    if (h->h2d) cudaStreamSynchronize(h->h2d);
    if (h->d2h) cudaStreamSynchronize(h->d2h);
    for (int k = 0; k < dslash_s::kSlots; ++k) {
        if (h->slot_in[k]) cudaFree(h->slot_in[k]);
        if (h->slot_out[k]) cudaFree(h->slot_out[k]);
        for (cudaEvent_t e : {h->ev_in_ready[k], h->ev_in_free[k], h->ev_out_ready[k], h->ev_out_free[k]})
            if (e) cudaEventDestroy(e);
    }
    if (h->ev_batch) cudaEventDestroy(h->ev_batch);
    for (void* q : h->ipc_opened) cudaIpcCloseMemHandle(q);
    if (h->ctl) cudaFree(h->ctl);
    for (char* q : h->lslab)
        if (q) cudaFree(q);
    if (h->cg_dd) cudaFree(h->cg_dd);
    for (void* v : h->cg_vec32)
        if (v) cudaFree(v);
    for (void* v : h->links32)
        if (v) cudaFree(v);
    for (void* v : h->cgm_vec)
        if (v) cudaFree(v);
    if (h->cgm_small) cudaFree(h->cgm_small);
    for (void* v : h->cg_vec)
        if (v) cudaFree(v);
    if (h->cg_partial) cudaFree(h->cg_partial);
    if (h->cg_scalar) cudaFree(h->cg_scalar);
    if (h->cg_partial2) cudaFree(h->cg_partial2);
    if (h->cg_bar) cudaFree(h->cg_bar);
    if (h->cg_host_rr) cudaFreeHost(h->cg_host_rr);
    for (cudaEvent_t e : h->cg_ev)
        if (e) cudaEventDestroy(e);
    if (h->h2d) cudaStreamDestroy(h->h2d);
    if (h->d2h) cudaStreamDestroy(h->d2h);
    for (auto& t : h->tpool) {
        cudaEventDestroy(t.a);
        cudaEventDestroy(t.b);
    }
    if (h->nccl) ncclCommDestroy(h->nccl);
    if (h->ev_start) cudaEventDestroy(h->ev_start);
    if (h->ev_halo) cudaEventDestroy(h->ev_halo);
    if (h->comm) cudaStreamDestroy(h->comm);
    if (h->ev_bdone) cudaEventDestroy(h->ev_bdone);
    delete h;
    return DSLASH_OK;
}

extern "C" const char* dslash_error_string(dslash_t h) {
    if (!h) return g_last_error.c_str();
    return h->msg.c_str();
}
