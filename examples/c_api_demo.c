/*
 * c_api_demo.c -- the HISQ Dslash library used from plain C through include/hisq_dslash.h
 * (no Python, no PyTorch).  Builds random links and vectors on the host, loads the links,
 * applies D_eo and D_oe from host buffers (dslash_apply_host), and checks the
 * anti-Hermiticity identity <chi_e, D_eo psi_o> = -<D_oe chi_e, psi_o> (Eq. (1):
 * the backward terms are the adjoints of the forward ones).  Prints one line and exits 0 on
 * success.
 *
 *   cc -O2 examples/c_api_demo.c -I include -L paper_conf_sc_dufekgaad024_b200 -lhisq_dslash -lm
 *   ./c_api_demo [Lx Ly Lz Lt]
 */
#include <complex.h>
#include <math.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include "hisq_dslash.h"

static uint64_t state = 0x9E3779B97F4A7C15ull;
static double uniform(void) {  /* xorshift64*, deterministic */
    state ^= state >> 12;
    state ^= state << 25;
    state ^= state >> 27;
    return ((state * 0x2545F4914F6CDD1Dull) >> 11) * (1.0 / 9007199254740992.0);
}
static double complex gauss(void) {
    const double u1 = uniform() + 1e-300, u2 = uniform();
    const double r = sqrt(-2.0 * log(u1));
    return r * cos(6.283185307179586 * u2) + I * r * sin(6.283185307179586 * u2);
}

#define CHECK(call)                                                                              \
    do {                                                                                         \
        dslash_status st_ = (call);                                                              \
        if (st_ != DSLASH_OK) {                                                                  \
            fprintf(stderr, "%s failed (%d): %s\n", #call, (int)st_, dslash_error_string(h));    \
            return 1;                                                                            \
        }                                                                                        \
    } while (0)

int main(int argc, char** argv) {
    int32_t dims[4] = {8, 8, 8, 16};
    const int32_t grid[4] = {1, 1, 1, 1};
    if (argc == 5)
        for (int d = 0; d < 4; ++d) dims[d] = atoi(argv[1 + d]);
    const int64_t V = (int64_t)dims[0] * dims[1] * dims[2] * dims[3];
    dslash_t h = NULL;
    CHECK(dslash_create(dims, grid, DSLASH_BOTH, DSLASH_F64, NULL, 1, 0, &h));
    const int64_t vh = dslash_local_half_volume(h);
    double complex* fat = malloc(sizeof(double complex) * V * 36);
    double complex* lng = malloc(sizeof(double complex) * V * 36);
    double complex* psi = malloc(sizeof(double complex) * 3 * vh);   /* odd source  */
    double complex* chi = malloc(sizeof(double complex) * 3 * vh);   /* even vector */
    double complex* dpsi = malloc(sizeof(double complex) * 3 * vh);
    double complex* dchi = malloc(sizeof(double complex) * 3 * vh);
    if (!fat || !lng || !psi || !chi || !dpsi || !dchi) return 2;
    for (int64_t i = 0; i < V * 36; ++i) {  /* general (non-unitary) links: nothing assumes SU(3) */
        fat[i] = gauss();
        lng[i] = 0.25 * gauss();
    }
    for (int64_t i = 0; i < 3 * vh; ++i) {
        psi[i] = gauss();
        chi[i] = gauss();
    }
    CHECK(dslash_load_links(h, fat, lng, 0, NULL));
    CHECK(dslash_apply_host(h, dpsi, psi, DSLASH_EVEN, NULL));  /* D_eo psi_o */
    CHECK(dslash_apply_host(h, dchi, chi, DSLASH_ODD, NULL));   /* D_oe chi_e */
    CHECK(dslash_sync(h));
    double complex lhs = 0, rhs = 0;
    double nchi = 0, ndpsi = 0;
    for (int64_t i = 0; i < 3 * vh; ++i) {
        lhs += conj(chi[i]) * dpsi[i];
        rhs -= conj(dchi[i]) * psi[i];
        nchi += creal(conj(chi[i]) * chi[i]);
        ndpsi += creal(conj(dpsi[i]) * dpsi[i]);
    }
    const double rel = cabs(lhs - rhs) / sqrt(nchi * ndpsi);
    printf("c_api_demo: dims %dx%dx%dx%d Vh=%lld <chi,D psi>=%.6e%+.6ei  -<D chi,psi>=%.6e%+.6ei  rel.diff=%.2e\n",
           dims[0], dims[1], dims[2], dims[3], (long long)vh, creal(lhs), cimag(lhs), creal(rhs), cimag(rhs), rel);
    CHECK(dslash_destroy(h));
    free(fat);
    free(lng);
    free(psi);
    free(chi);
    free(dpsi);
    free(dchi);
    return rel < 1e-12 ? 0 : 3;
}
