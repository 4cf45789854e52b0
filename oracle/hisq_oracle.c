/*
 * hisq_oracle.c -- plain, slow, obviously-correct CPU oracle of the single-parity
 * improved-staggered (HISQ) Dslash.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The CUDA product
 * path never calls it, and it shares no code with the CUDA path (the only shared
 * module is the seeded input generator fieldgen/).
 *
 * What it computes (§II, Eq. (1); Naik third-neighbour terms per
 * L27 §I and L51 "first- and third-nearest neighbor terms"; readings Z1, Z2, Z4,
 * Z5, Z6, Z10 of DESIGN.md):  for every site x of parity p(x) = parity,
 *
 *   chi(x) = sum_{mu=0..3} [  F(x,mu)        psi(x+mu)
 *                           - F(x-mu,mu)^dag  psi(x-mu)
 *                           + N(x,mu)         psi(x+3mu)
 *                           - N(x-3mu,mu)^dag psi(x-3mu) ]
 *
 * with coordinates taken modulo the lattice extents (periodic), (A^dag)_{ij} =
 * conj(A_{ji}), no phases (they are folded into the links) and no 1/2 factor.
 * The adjoint back-links are formed on the fly from the forward links, the target
 * sites are visited in lexicographic order, mu ascending, terms in the order
 * above.  Pins: tests/test_oracle_pins.py (P1-P9 of DESIGN.md).
 *
 * Layouts (all complex = C99 double complex):
 *   dims = {Lx, Ly, Lz, Lt}, lex(x,y,z,t) = x + Lx*(y + Ly*(z + Lz*t));
 *   fat, lng: [lex][mu][3][3]   (|i|x|j| complex matrices, L^4 x |k|)
 *   psi, chi: [lex][3]          (full lattice; psi is read only at parity 1-parity,
 *                                chi is written at every site: 0 off the target parity)
 *
 * Build: gcc -O2 -ffp-contract=off (no fast-math); OpenMP over target sites is
 * allowed because sites are independent, so results do not depend on threads.
 */
#include <complex.h>
#include <stdint.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define ORACLE_API __attribute__((visibility("default")))

typedef double complex cplx;

static int64_t lex_of(const int32_t d[4], int64_t x, int64_t y, int64_t z, int64_t t) {
    return x + d[0] * (y + d[1] * (z + d[2] * t));
}

/* coordinate c of lex index s */
static void coords_of(const int32_t d[4], int64_t s, int64_t c[4]) {
    c[0] = s % d[0]; s /= d[0];
    c[1] = s % d[1]; s /= d[1];
    c[2] = s % d[2]; s /= d[2];
    c[3] = s;
}

/* lex index of the site c + h * e_mu, periodic */
static int64_t hop(const int32_t d[4], const int64_t c[4], int mu, int64_t h) {
    int64_t n[4] = {c[0], c[1], c[2], c[3]};
    n[mu] = ((n[mu] + h) % d[mu] + d[mu]) % d[mu];
    return lex_of(d, n[0], n[1], n[2], n[3]);
}

/* r += A v   (A = link at site s, direction mu) */
static void add_mv(cplx r[3], const cplx* links, int64_t s, int mu, const cplx* psi, int64_t src) {
    const cplx* A = links + 9 * (4 * s + mu);
    const cplx* v = psi + 3 * src;
    for (int i = 0; i < 3; ++i) {
        cplx acc = 0;
        for (int j = 0; j < 3; ++j) acc += A[3 * i + j] * v[j];
        r[i] += acc;
    }
}

/* r -= A^dag v   (A = link at site s, direction mu), (A^dag)_{ij} = conj(A_{ji}) */
static void sub_adj_mv(cplx r[3], const cplx* links, int64_t s, int mu, const cplx* psi, int64_t src) {
    const cplx* A = links + 9 * (4 * s + mu);
    const cplx* v = psi + 3 * src;
    for (int i = 0; i < 3; ++i) {
        cplx acc = 0;
        for (int j = 0; j < 3; ++j) acc += conj(A[3 * j + i]) * v[j];
        r[i] -= acc;
    }
}

/* chi(x) for one site x (lex index s) */
static void oracle_site(const int32_t d[4], const cplx* fat, const cplx* lng, const cplx* psi, int64_t s,
                        cplx out[3]) {
    int64_t c[4];
    coords_of(d, s, c);
    cplx r[3] = {0, 0, 0};
    for (int mu = 0; mu < 4; ++mu) {
        add_mv(r, fat, s, mu, psi, hop(d, c, mu, +1));                           /* + F(x,mu) psi(x+mu)        */
        sub_adj_mv(r, fat, hop(d, c, mu, -1), mu, psi, hop(d, c, mu, -1));       /* - F(x-mu,mu)^dag psi(x-mu)  */
        add_mv(r, lng, s, mu, psi, hop(d, c, mu, +3));                           /* + N(x,mu) psi(x+3mu)        */
        sub_adj_mv(r, lng, hop(d, c, mu, -3), mu, psi, hop(d, c, mu, -3));       /* - N(x-3mu,mu)^dag psi(x-3mu) */
    }
    out[0] = r[0];
    out[1] = r[1];
    out[2] = r[2];
}

static int dims_ok(const int32_t d[4]) {
    for (int i = 0; i < 4; ++i)
        if (d[i] < 1) return 0;
    return 1;
}

/*
 * Full-lattice apply: chi[x] = (D psi)(x) for p(x) = parity, chi[x] = 0 otherwise.
 * nthreads <= 0: OpenMP default; 1: single-threaded.  Returns 0, or -1 on bad args.
 */
ORACLE_API int oracle_dslash(const int32_t dims[4], const cplx* fat, const cplx* lng, const cplx* psi, cplx* chi,
                             int32_t parity, int32_t nthreads) {
    if (!dims_ok(dims) || !fat || !lng || !psi || !chi || (parity & ~1)) return -1;
    const int64_t V = (int64_t)dims[0] * dims[1] * dims[2] * dims[3];
#ifdef _OPENMP
    const int nt = nthreads > 0 ? nthreads : omp_get_num_procs();
#pragma omp parallel for schedule(static) num_threads(nt)
#endif
    for (int64_t s = 0; s < V; ++s) {
        int64_t c[4];
        coords_of(dims, s, c);
        if (((c[0] + c[1] + c[2] + c[3]) & 1) != parity) {
            chi[3 * s] = chi[3 * s + 1] = chi[3 * s + 2] = 0;
            continue;
        }
        oracle_site(dims, fat, lng, psi, s, chi + 3 * s);
    }
    (void)nthreads;
    return 0;
}

/*
 * Sampled apply: out[k][3] = (D psi)(sites[k]) for k < nsites, each site a lex
 * index (any parity).  Used to check full-size GPU outputs site by site.
 */
ORACLE_API int oracle_dslash_sites(const int32_t dims[4], const cplx* fat, const cplx* lng, const cplx* psi,
                                   int64_t nsites, const int64_t* sites, cplx* out, int32_t nthreads) {
    if (!dims_ok(dims) || !fat || !lng || !psi || !out || (nsites > 0 && !sites) || nsites < 0) return -1;
    const int64_t V = (int64_t)dims[0] * dims[1] * dims[2] * dims[3];
    for (int64_t k = 0; k < nsites; ++k)
        if (sites[k] < 0 || sites[k] >= V) return -1;
#ifdef _OPENMP
    const int nt = nthreads > 0 ? nthreads : omp_get_num_procs();
#pragma omp parallel for schedule(static) num_threads(nt)
#endif
    for (int64_t k = 0; k < nsites; ++k) oracle_site(dims, fat, lng, psi, sites[k], out + 3 * k);
    (void)nthreads;
    return 0;
}
