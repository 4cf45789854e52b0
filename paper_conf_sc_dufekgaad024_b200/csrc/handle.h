// handle.h -- the library handle and the host-side helpers shared by dslash_lib.cu and solver.cu.
#pragma once

#include <cuda_runtime.h>
#include <nccl.h>

#include <string>
#include <vector>

#include "hisq_dslash.h"
#include "dispatch.h"

// P2P transport control block (device memory, CUDA-IPC-exported; every rank maps every other
// rank's block).  Flags are epoch counters written by stream memory operations
// (cuStreamWriteValue32) and waited on with cuStreamWaitValue32 (GEQ).
constexpr int kMaxRanks = 64;
struct P2PControl {
    // [0..7] ready[d][side]: written by the neighbour that fills my ghost[d][side];
    // [8..15] free_from[d][side]: written by the neighbour whose ghost my bottom (side 0) / top
    //         (side 1) face fills, once it consumed it;
    // [16..19] lslab_ready[d]: my minus neighbour filled my link-slab buffer of direction d;
    // [20..23] lslab_free[d]: my plus neighbour converted the link slab I sent it
    unsigned int flags[32];
    // cross-rank reduction (dslash_cg without NCCL): rank r's double-double partial of reduction
    // e lands in red_val[e & 1][r] and then red_flag[r] = e
    unsigned int red_flag[kMaxRanks];
    double2 red_val[2][kMaxRanks];
};

struct dslash_s {
    dslash_plan_t plan{};
    int32_t global_dims[4]{}, proc_grid[4]{};
    int parity_mask = 0, precision = 0, device = 0;
    int kernel = DSLASH_KERNEL_DIR2, block = 0, force_halo = 0, overlap = 1, timing = 0, min_blocks = 0;
    int recon = 18;
    double long_inv_scale = 1.0;
    double long_scale = 1.0;        // recon-9: s of N = s e^{i psi} W
    size_t link_bytes = 0;
    bool loaded = false;
    void* links[2] = {nullptr, nullptr};
    char* ghost[4][2] = {};        // source-vector ghost faces [nrhs][3][face_vh]
    char* zsend[2] = {};           // packed z faces to send (NCCL path)
    int ghost_rhs = 0;             // number of right-hand sides the ghost buffers hold
    void* stage_in = nullptr;      // apply_host staging
    void* stage_out = nullptr;
    static constexpr int kSlots = 3;  // apply_host_batch pipeline depth
    void* slot_in[kSlots] = {};
    void* slot_out[kSlots] = {};
    cudaStream_t h2d = nullptr, d2h = nullptr;
    cudaEvent_t ev_in_ready[kSlots] = {}, ev_in_free[kSlots] = {}, ev_out_ready[kSlots] = {},
                ev_out_free[kSlots] = {}, ev_batch = nullptr;
    cudaStream_t comm = nullptr;
    cudaEvent_t ev_start = nullptr, ev_halo = nullptr, ev_bdone = nullptr;
    bool halo_pending = false;
    ncclComm_t nccl = nullptr;
    struct TimedLaunch {
        cudaEvent_t a, b;
        int kind;
    };
    std::vector<TimedLaunch> tpool;
    size_t tused = 0;
    // conjugate-gradient scratch (solver.cu): r, p, q on the target parity, t on the other one,
    // block partial sums and the reduced scalars
    void* cg_vec[4] = {};
    // dslash_cg_multi_blocked scratch (solver_multi.cu): r, p, q, t of cgm_bytes each, grown on demand,
    // and its partials / scalars / convergence record
    void* cgm_vec[4] = {};
    size_t cgm_bytes = 0;
    void* cgm_small = nullptr;
    // mixed-precision solver (dslash_cg_mixed): fp32 e, r, p, q, t and the fp32 links per parity
    void* cg_vec32[5] = {};
    void* links32[2] = {};
    double2* cg_partial = nullptr;      // block partials, double-double
    double* cg_scalar = nullptr;
    double2* cg_dd = nullptr;           // [0] this rank's sum, [1 + r] rank r's (ncclAllGather)
    // fused CG step (one rank): the |r|^2 block partials and the grid-barrier counter with the
    // arrivals expected by the end of the next launch's barrier
    double2* cg_partial2 = nullptr;
    unsigned long long* cg_bar = nullptr;
    unsigned long long cg_bar_next = 0;
    int cg_fused = -1;  // -1: not probed yet; 0: cooperative launch unavailable; 1: fused step
    // CG host side, kept across solves (pinned allocation and event creation cost more than a
    // short solve): <r,r> per iteration, pinned; events of the lagged convergence check
    double* cg_host_rr = nullptr;
    int cg_host_cap = 0;
    cudaEvent_t cg_ev[4] = {};
    int pdl = 1;                        // programmatic dependent launch of the stencil kernels
    unsigned int epoch = 0;             // halo exchanges started so far (P2P epoch flags)
    // P2P transport (DSLASH_TRANSPORT_P2P): CUDA-IPC-mapped neighbour buffers, copy engines and
    // stream memory operations.  flags (device, IPC-exported): [0..7] ready[d][side] (written by the
    // neighbour that fills my ghost[d][side]), [8..15] free_from[d][side] (written by the neighbour
    // whose ghost my bottom (side 0) / top (side 1) face fills, once it consumed it).
    int transport = DSLASH_TRANSPORT_NCCL;
    int halo_dryrun = 0;                // DSLASH_OPT_HALO_DRYRUN (timing aid: exchange moves no bytes)
    int stage = 0;                      // DSLASH_OPT_STAGE: neighbour-staged kernel (x/y rows in smem by TMA)
    int self_nccl = 0;                  // DSLASH_OPT_SELF_NCCL: self-neighbour faces via NCCL
    P2PControl* ctl = nullptr;          // my control block (IPC-exported)
    unsigned int* flags = nullptr;      // = ctl->flags
    std::vector<P2PControl*> peer_ctl;  // every rank's control block (mine at [rank])
    // link halo under P2P (dslash_load_links): the minus neighbour copies its top 3 link slices
    // straight into lslab[d] ([fat | long], canonical slab layout), then raises my
    // lslab_ready[d]; load_links_count numbers those exchanges
    char* lslab[4] = {};
    size_t lslab_bytes[4] = {};         // bytes of ONE kind (fat or long) in lslab[d]
    char* peer_lslab[4] = {};           // my plus neighbour's lslab[d]
    unsigned int link_epoch = 0;
    unsigned int red_epoch = 0;         // cross-rank reductions so far
    char* peer_ghost[4][2] = {};        // [d][0]: minus nbr's plus ghost; [d][1]: plus nbr's minus ghost
    unsigned int* peer_ready[4][2] = {};  // the ready flag of that ghost
    unsigned int* peer_free[4][2] = {};   // [d][0]: minus nbr's free_from[d][1]; [d][1]: plus nbr's free_from[d][0]
    std::vector<void*> ipc_opened;
    bool p2p_ready = false;
    // producer push (DSLASH_OPT_PUSH, P2P transport): the ghosts hold two banks (epoch e reads bank
    // e & 1); an apply_push of epoch e stores the faces of its output straight into the neighbours'
    // bank (e + 1) & 1 from the stencil kernel's epilogue, so the next apply (epoch e + 1, source =
    // that output) exchanges no bytes
    int push = 0;
    size_t ghost_bank[4] = {};          // bytes from bank 0 to bank 1 of ghost[d][side]
    const void* pushed_src = nullptr;   // the vector whose faces were pushed for epoch pushed_epoch
    unsigned int pushed_epoch = 0;      // 0: none pending
    int pushed_rhs = 0;
    dslash_status err = DSLASH_OK;
    std::string msg;
};

// Every entry point that touches the GPU runs on the handle's device (several handles on several
// devices in one process) and restores the caller's current device on return.
struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(const dslash_s* h) {
        int cur = 0;
        if (h && cudaGetDevice(&cur) == cudaSuccess && cur != h->device && cudaSetDevice(h->device) == cudaSuccess)
            prev = cur;
    }
    ~DeviceGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

// Record a failure on the handle (first error wins) or, with h == NULL, in the thread's last
// error; returns st.
dslash_status hisq_fail(dslash_t h, dslash_status st, const char* fmt, ...);

#define CU(h, call)                                                                                   \
    do {                                                                                              \
        cudaError_t e_ = (call);                                                                      \
        if (e_ != cudaSuccess)                                                                        \
            return hisq_fail((h), e_ == cudaErrorMemoryAllocation ? DSLASH_ERR_OOM : DSLASH_ERR_CUDA, \
                             "%s:%d %s: %s", __FILE__, __LINE__, #call, cudaGetErrorString(e_));      \
    } while (0)

#define NC(h, call)                                                                                   \
    do {                                                                                              \
        ncclResult_t r_ = (call);                                                                     \
        if (r_ != ncclSuccess)                                                                        \
            return hisq_fail((h), DSLASH_ERR_NCCL, "%s:%d %s: %s", __FILE__, __LINE__, #call,         \
                             ncclGetErrorString(r_));                                                 \
    } while (0)

// Producer push from a vector kernel (the CG direction update p = r + beta p): the element of
// colour c at cb of a site within 3 slices of a pushed face is also stored into the neighbour's
// ghost bank, in the face order of the stencil kernel's push (stencil.cuh).
struct FacePush {
    void* dst[4][2];      // [mu][side] peer ghost banks, [3][face_vh[mu]] (only where mask has mu)
    int mask;             // bit mu: push direction mu (2 = z, 3 = t)
    int64_t vh, face_vh[4];
    int lxh, L1, L2, L3;  // local extents (lxh = Lx / 2)
};
// before the pushing kernel on stream s: wait for the neighbours' releases, fill *fp (mask 0 when
// the handle does not push or has no halo); after it: raise the neighbours' ready flags
dslash_status hisq_push_begin(dslash_t h, cudaStream_t s, FacePush* fp);
dslash_status hisq_push_end(dslash_t h, cudaStream_t s, const void* out);
// drop pushed faces no apply will consume (the CG's last direction update): the pushed epoch is
// retired as if an apply had consumed it, on every rank alike
dslash_status hisq_push_discard(dslash_t h, cudaStream_t s);

// P2P transport, several ranks: copy this rank's double-double `mine` (device) into slot
// [rank] of every rank's control block, raise their flags, and make stream s wait until every
// rank's value has arrived in mine; *all = my control block's slots (nranks values, rank order)
dslash_status hisq_p2p_gather(dslash_t h, cudaStream_t s, const double2* mine, const double2** all);

// round the fp64 internal links of `parity` into h->links32[parity] (fp32 paired layout)
dslash_status hisq_convert_links_sloppy(dslash_t h, int parity);

// out = D in on target parity `parity` for nrhs back-to-back vectors (dslash_lib.cu); push: also
// push the faces of out into the neighbours' ghosts for the next apply (DSLASH_OPT_PUSH)
dslash_status hisq_apply(dslash_t h, void* out, const void* in, int32_t parity, int32_t nrhs, cudaStream_t s,
                         bool push = false);
// the same on site-blocked vectors (dslash_apply_multi_blocked)
dslash_status hisq_apply_blocked(dslash_t h, void* out, const void* in, int32_t parity, int32_t nrhs, cudaStream_t s);
