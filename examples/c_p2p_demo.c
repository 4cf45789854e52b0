/*
 * c_p2p_demo.c -- a multi-rank P2P partition driven from plain C (no Python, no PyTorch, no
 * MPI): the whole multi-GPU set-up the C ABI owns (include/hisq_dslash.h, DSLASH_TRANSPORT_P2P).
 *
 * The parent forks NRANKS child processes before touching CUDA.  Child r is rank r of a
 * t-partitioned lattice (proc_grid {1,1,1,NRANKS}, the north star's first split direction), on
 * device r % ndev (all on device 0 with one GPU: several ranks per GPU work with P2P).  The
 * children
 *   1. create a handle (nranks > 1 and no NCCL id selects the P2P transport),
 *   2. publish their IPC blobs in a shared anonymous mapping, meet at a process-shared barrier,
 *      and open everyone's blobs,
 *   3. load their LOCAL forward links: dslash_load_links fetches the 3 link slices below each
 *      partition face from the minus neighbour itself (copy engines into the IPC-mapped slab
 *      buffers, epoch flags) -- the caller exchanges nothing,
 *   4. apply D (dslash_apply_host: halo exchange into the neighbours' ghosts, interior +
 *      boundary kernels) for both parities and write their part of chi into the shared mapping.
 * Then rank 0 applies D on the WHOLE lattice with one rank and checks that the gathered N-rank
 * result is bitwise identical (same per-site arithmetic), and that the
 * anti-Hermiticity identity <chi_e, D_eo psi_o> = -<D_oe chi_e, psi_o> holds.
 * Fields are generated from global coordinates, so every rank sees its slice of one global field.
 *
 *   cc -O2 examples/c_p2p_demo.c -I include -L paper_conf_sc_dufekgaad024_b200 -lhisq_dslash -lpthread -lm
 *   ./c_p2p_demo [NRANKS Lx Ly Lz Lt_global]      (default 2 8 8 8 16)
 */
#define _GNU_SOURCE
#include <complex.h>
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>
#include <sys/wait.h>
#include <unistd.h>

#include "hisq_dslash.h"

/* counter-based Gaussian keyed by (stream, global index): the same value on every rank */
static uint64_t mix(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
static double unit(uint64_t k) { return ((mix(k) >> 11) + 0.5) * (1.0 / 9007199254740992.0); }
static double complex gauss(uint64_t stream, uint64_t idx) {
    const uint64_t k = mix(stream * 0x100000001B3ull + idx) * 2;
    const double r = sqrt(-2.0 * log(unit(k))), th = 6.283185307179586 * unit(k + 1);
    return r * cos(th) + I * r * sin(th);
}

typedef struct {
    pthread_barrier_t bar;
    int failed;
} shared_hdr;

static int32_t G[4] = {8, 8, 8, 16};
static int nranks = 2;

/* links of the local box [t0, t0 + lt): canonical [t][z][y][x][mu][3][3], keyed by global site */
static void make_links(double complex* fat, double complex* lng, int t0, int lt) {
    int64_t i = 0;
    for (int t = t0; t < t0 + lt; ++t)
        for (int z = 0; z < G[2]; ++z)
            for (int y = 0; y < G[1]; ++y)
                for (int x = 0; x < G[0]; ++x) {
                    const uint64_t g = (uint64_t)x + G[0] * ((uint64_t)y + G[1] * ((uint64_t)z + G[2] * (uint64_t)t));
                    for (int e = 0; e < 36; ++e, ++i) {
                        fat[i] = gauss(1, g * 36 + e);
                        lng[i] = 0.25 * gauss(2, g * 36 + e);
                    }
                }
}

/* a vector on `parity` of the local box, [3][vh] (cb = local lex / 2), keyed by global site */
static void make_vector(double complex* v, int parity, int t0, int lt, uint64_t stream) {
    const int64_t vh = (int64_t)G[0] * G[1] * G[2] * lt / 2;
    int64_t cb = 0;
    for (int t = t0; t < t0 + lt; ++t)
        for (int z = 0; z < G[2]; ++z)
            for (int y = 0; y < G[1]; ++y)
                for (int x = 0; x < G[0]; ++x) {
                    if (((x + y + z + t) & 1) != parity) continue;
                    const uint64_t g = (uint64_t)x + G[0] * ((uint64_t)y + G[1] * ((uint64_t)z + G[2] * (uint64_t)t));
                    for (int c = 0; c < 3; ++c) v[c * vh + cb] = gauss(stream, g * 3 + c);
                    ++cb;
                }
}

#define CHECK(call)                                                                              \
    do {                                                                                         \
        dslash_status st_ = (call);                                                              \
        if (st_ != DSLASH_OK) {                                                                  \
            fprintf(stderr, "rank %d: %s failed (%d): %s\n", rank, #call, (int)st_,             \
                    dslash_error_string(h));                                                     \
            hdr->failed = 1;                                                                     \
            return 1;                                                                            \
        }                                                                                        \
    } while (0)

/* shared mapping: header | blobs[nranks] | chi_e[3][Vh] | chi_o[3][Vh] (global cb order) */
static int rank_main(int rank, shared_hdr* hdr, char* blobs, double complex* out_e, double complex* out_o) {
    dslash_t h = NULL;
    const int ndev = dslash_device_count();
    if (ndev < 1) {
        fprintf(stderr, "rank %d: no CUDA device\n", rank);
        hdr->failed = 1;
        return 1;
    }
    CHECK(dslash_set_device(rank % ndev));
    const int32_t grid[4] = {1, 1, 1, nranks};
    CHECK(dslash_create(G, grid, DSLASH_BOTH, DSLASH_F64, NULL, nranks, rank, &h));
    const int64_t bsz = dslash_ipc_blob_size();
    CHECK(dslash_get_ipc_blob(h, blobs + rank * bsz));
    pthread_barrier_wait(&hdr->bar);                       /* every blob published */
    if (hdr->failed) return 1;
    CHECK(dslash_open_ipc_blobs(h, blobs));
    const int lt = G[3] / nranks, t0 = rank * lt;
    const int64_t V = (int64_t)G[0] * G[1] * G[2] * lt, vh = V / 2;
    double complex* fat = malloc(sizeof(double complex) * V * 36);
    double complex* lng = malloc(sizeof(double complex) * V * 36);
    double complex* src = malloc(sizeof(double complex) * 3 * vh);
    double complex* dst = malloc(sizeof(double complex) * 3 * vh);
    if (!fat || !lng || !src || !dst) return 2;
    make_links(fat, lng, t0, lt);
    CHECK(dslash_load_links(h, fat, lng, 0, NULL));        /* link halo from the minus neighbour */
    for (int p = 0; p < 2; ++p) {
        make_vector(src, 1 - p, t0, lt, 3 + p);
        CHECK(dslash_apply_host(h, dst, src, p, NULL));    /* halo exchange + interior + boundary */
        CHECK(dslash_sync(h));
        double complex* out = p ? out_o : out_e;
        const int64_t vh_glob = vh * nranks;
        for (int c = 0; c < 3; ++c) memcpy(out + c * vh_glob + rank * vh, dst + c * vh, sizeof(double complex) * vh);
    }
    pthread_barrier_wait(&hdr->bar);                       /* every rank applied: now tear down */
    CHECK(dslash_destroy(h));
    free(fat);
    free(lng);
    free(src);
    free(dst);
    return 0;
}

/* rank 0, after the partitioned run: the same applies on the whole lattice with one rank */
static int check_single(shared_hdr* hdr, const double complex* out_e, const double complex* out_o) {
    const int rank = 0;
    dslash_t h = NULL;
    CHECK(dslash_set_device(0));
    const int32_t one[4] = {1, 1, 1, 1};
    CHECK(dslash_create(G, one, DSLASH_BOTH, DSLASH_F64, NULL, 1, 0, &h));
    const int64_t V = (int64_t)G[0] * G[1] * G[2] * G[3], vh = V / 2;
    double complex* fat = malloc(sizeof(double complex) * V * 36);
    double complex* lng = malloc(sizeof(double complex) * V * 36);
    double complex* src[2] = {malloc(sizeof(double complex) * 3 * vh), malloc(sizeof(double complex) * 3 * vh)};
    double complex* dst = malloc(sizeof(double complex) * 3 * vh);
    make_links(fat, lng, 0, G[3]);
    CHECK(dslash_load_links(h, fat, lng, 0, NULL));
    int equal = 1;
    for (int p = 0; p < 2; ++p) {
        make_vector(src[p], 1 - p, 0, G[3], 3 + p);
        CHECK(dslash_apply_host(h, dst, src[p], p, NULL));
        CHECK(dslash_sync(h));
        if (memcmp(dst, p ? out_o : out_e, sizeof(double complex) * 3 * vh)) equal = 0;
    }
    /* <chi_e, D_eo psi_o> = -<D_oe chi_e, psi_o>: src[0] = psi_o, src[1] = chi_e */
    double complex lhs = 0, rhs = 0;
    double n1 = 0, n2 = 0;
    for (int64_t i = 0; i < 3 * vh; ++i) {
        lhs += conj(src[1][i]) * out_e[i];
        rhs -= conj(out_o[i]) * src[0][i];
        n1 += creal(conj(src[1][i]) * src[1][i]);
        n2 += creal(conj(out_e[i]) * out_e[i]);
    }
    const double rel = cabs(lhs - rhs) / sqrt(n1 * n2);
    printf("c_p2p_demo: %d ranks, global %dx%dx%dx%d t-partitioned over P2P, link halo in load_links: "
           "gathered chi %s the 1-rank chi bitwise; anti-Hermiticity rel.diff=%.2e\n",
           nranks, G[0], G[1], G[2], G[3], equal ? "EQUALS" : "DIFFERS FROM", rel);
    fflush(stdout);  /* the child leaves with _exit, which does not flush stdio */
    CHECK(dslash_destroy(h));
    free(fat);
    free(lng);
    free(src[0]);
    free(src[1]);
    free(dst);
    return (equal && rel < 1e-12) ? 0 : 3;
}

int main(int argc, char** argv) {
    if (argc == 6) {
        nranks = atoi(argv[1]);
        for (int d = 0; d < 4; ++d) G[d] = atoi(argv[2 + d]);
    }
    if (nranks < 2 || G[3] % nranks) {
        fprintf(stderr, "usage: %s NRANKS Lx Ly Lz Lt (NRANKS >= 2 divides Lt)\n", argv[0]);
        return 2;
    }
    const int64_t vh_glob = (int64_t)G[0] * G[1] * G[2] * G[3] / 2;
    const size_t bsz = (size_t)dslash_ipc_blob_size();   /* host-only: no CUDA call */
    const size_t bytes = 4096 + bsz * nranks + 2 * sizeof(double complex) * 3 * vh_glob;
    char* base = mmap(NULL, bytes, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_ANONYMOUS, -1, 0);
    if (base == MAP_FAILED) return 2;
    shared_hdr* hdr = (shared_hdr*)base;
    pthread_barrierattr_t at;
    pthread_barrierattr_init(&at);
    pthread_barrierattr_setpshared(&at, PTHREAD_PROCESS_SHARED);
    pthread_barrier_init(&hdr->bar, &at, (unsigned)nranks);
    hdr->failed = 0;
    char* blobs = base + 4096;
    double complex* out_e = (double complex*)(blobs + bsz * nranks);
    double complex* out_o = out_e + 3 * vh_glob;
    pid_t pid[64];
    for (int r = 0; r < nranks && r < 64; ++r) {
        pid[r] = fork();
        if (pid[r] == 0) _exit(rank_main(r, hdr, blobs, out_e, out_o));
    }
    int bad = 0;
    for (int r = 0; r < nranks && r < 64; ++r) {
        int status = 0;
        waitpid(pid[r], &status, 0);
        if (!WIFEXITED(status) || WEXITSTATUS(status)) bad = 1;
    }
    if (bad || hdr->failed) {
        fprintf(stderr, "c_p2p_demo: a rank failed\n");
        return 1;
    }
    /* the 1-rank reference in a fresh child too (this process never initialises CUDA) */
    pid_t c = fork();
    if (c == 0) _exit(check_single(hdr, out_e, out_o));
    int status = 0;
    waitpid(c, &status, 0);
    return WIFEXITED(status) ? WEXITSTATUS(status) : 1;
}
