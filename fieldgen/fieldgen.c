/*
 * fieldgen.c -- seeded, counter-based synthetic input fields for the HISQ Dslash.
 *
 * This module is the ONLY code shared between the CPU oracle (oracle/) and the
 * CUDA product path (paper_conf_sc_dufekgaad024_b200/).  It holds none of the
 * Dslash arithmetic: it only draws random numbers and writes them in the layouts
 * the two sides consume.
 *
 * Workload recipe:
 *   - links: Haar-random SU(3) matrices (Gram-Schmidt of two complex Gaussian
 *     rows, third row = conj(row0 x row1), so det = 1), optionally scaled
 *     (long links use scale -1/24), or general complex Gaussian matrices;
 *   - source vector: i.i.d. complex Gaussian, unit variance per real component.
 *   Paper workload shape: 3x3 complex links per site and direction, one SU(3)
 *   colour vector per site (§II).
 *
 * Every number is a pure function of (seed, GLOBAL lexicographic site, slot,
 * element), so any partition of the global lattice regenerates exactly the same
 * global field (needed for the multi-GPU tests).
 *
 * Coordinates: global extents G = {Lx,Ly,Lz,Lt} (x fastest); a local box has
 * origin O and extents E.  global lex = x + Lx*(y + Ly*(z + Lz*t)).
 * Complex numbers are stored as interleaved (re, im) doubles.
 */
#include <math.h>
#include <stdint.h>
#include <string.h>

#define FG_API __attribute__((visibility("default")))

static inline uint64_t fg_mix(uint64_t z) {
    /* splitmix64 finaliser: a bijection on 64-bit words */
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

static inline uint64_t fg_key(uint64_t seed, uint64_t site, uint32_t slot, uint32_t n) {
    uint64_t h = fg_mix(seed ^ 0xD1B54A32D192ED03ull);
    h = fg_mix(h ^ site);
    h = fg_mix(h ^ (((uint64_t)slot << 32) | (uint64_t)n));
    return h;
}

/* uniform in the open interval (0,1) */
static inline double fg_u01(uint64_t h) { return ((double)(h >> 11) + 0.5) * (1.0 / 9007199254740992.0); }

/* one complex Gaussian, unit variance per real component (Box-Muller) */
static inline void fg_cgauss(uint64_t seed, uint64_t site, uint32_t slot, uint32_t n, double* re, double* im) {
    const double u1 = fg_u01(fg_key(seed, site, slot, 2u * n));
    const double u2 = fg_u01(fg_key(seed, site, slot, 2u * n + 1u));
    const double r = sqrt(-2.0 * log(u1));
    const double a = 6.283185307179586476925286766559 * u2;
    *re = r * cos(a);
    *im = r * sin(a);
}

/* Haar SU(3): rows 0,1 Gram-Schmidt-orthonormalised complex Gaussians,
 * row 2 = conj(row0 x row1).  m is [3][3] interleaved complex (row-major). */
static void fg_su3(uint64_t seed, uint64_t site, uint32_t slot, double* m) {
    double ar[3], ai[3], br[3], bi[3];
    for (int j = 0; j < 3; ++j) fg_cgauss(seed, site, slot, (uint32_t)j, &ar[j], &ai[j]);
    for (int j = 0; j < 3; ++j) fg_cgauss(seed, site, slot, (uint32_t)(3 + j), &br[j], &bi[j]);
    double n = 0.0;
    for (int j = 0; j < 3; ++j) n += ar[j] * ar[j] + ai[j] * ai[j];
    n = 1.0 / sqrt(n);
    for (int j = 0; j < 3; ++j) { ar[j] *= n; ai[j] *= n; }
    /* b -= <a,b> a, <a,b> = sum conj(a_j) b_j */
    double pr = 0.0, pi = 0.0;
    for (int j = 0; j < 3; ++j) {
        pr += ar[j] * br[j] + ai[j] * bi[j];
        pi += ar[j] * bi[j] - ai[j] * br[j];
    }
    for (int j = 0; j < 3; ++j) {
        br[j] -= pr * ar[j] - pi * ai[j];
        bi[j] -= pr * ai[j] + pi * ar[j];
    }
    n = 0.0;
    for (int j = 0; j < 3; ++j) n += br[j] * br[j] + bi[j] * bi[j];
    n = 1.0 / sqrt(n);
    for (int j = 0; j < 3; ++j) { br[j] *= n; bi[j] *= n; }
    /* c = conj(a x b) */
    double cr[3], ci[3];
    for (int j = 0; j < 3; ++j) {
        const int j1 = (j + 1) % 3, j2 = (j + 2) % 3;
        const double xr = (ar[j1] * br[j2] - ai[j1] * bi[j2]) - (ar[j2] * br[j1] - ai[j2] * bi[j1]);
        const double xi = (ar[j1] * bi[j2] + ai[j1] * br[j2]) - (ar[j2] * bi[j1] + ai[j2] * br[j1]);
        cr[j] = xr;
        ci[j] = -xi;
    }
    for (int j = 0; j < 3; ++j) {
        m[2 * (0 * 3 + j)] = ar[j]; m[2 * (0 * 3 + j) + 1] = ai[j];
        m[2 * (1 * 3 + j)] = br[j]; m[2 * (1 * 3 + j) + 1] = bi[j];
        m[2 * (2 * 3 + j)] = cr[j]; m[2 * (2 * 3 + j) + 1] = ci[j];
    }
}

static int fg_check_box(const int32_t G[4], const int32_t O[4], const int32_t E[4]) {
    for (int d = 0; d < 4; ++d) {
        if (G[d] < 1 || E[d] < 1 || O[d] < 0 || O[d] + E[d] > G[d]) return -1;
    }
    return 0;
}

static inline uint64_t fg_glex(const int32_t G[4], int64_t x, int64_t y, int64_t z, int64_t t) {
    return (uint64_t)(x + (int64_t)G[0] * (y + (int64_t)G[1] * (z + (int64_t)G[2] * t)));
}

/*
 * Matrix field over a local box: out[local lex][k][3][3] complex, k < nper.
 * kind 0 = Haar SU(3), kind 1 = complex Gaussian entries.  Every entry is
 * multiplied by `scale`.  With nper = 4 this is the canonical link layout
 * [t][z][y][x][mu][3][3] (|i|x|j| complex matrices, L^4 x |k|).
 * Returns the number of matrices written, or -1 on bad arguments.
 */
FG_API int64_t fg_matrices(const int32_t G[4], const int32_t O[4], const int32_t E[4], uint64_t seed,
                           int32_t nper, int32_t kind, double scale, double* out) {
    if (fg_check_box(G, O, E) || nper < 1 || (kind != 0 && kind != 1) || !out) return -1;
    const int64_t nloc = (int64_t)E[0] * E[1] * E[2] * E[3];
#pragma omp parallel for schedule(static)
    for (int64_t l = 0; l < nloc; ++l) {
        int64_t r = l;
        const int64_t x = r % E[0]; r /= E[0];
        const int64_t y = r % E[1]; r /= E[1];
        const int64_t z = r % E[2]; r /= E[2];
        const int64_t t = r;
        const uint64_t g = fg_glex(G, O[0] + x, O[1] + y, O[2] + z, O[3] + t);
        for (int k = 0; k < nper; ++k) {
            double* m = out + 18 * (l * nper + k);
            if (kind == 0) {
                fg_su3(seed, g, (uint32_t)k, m);
            } else {
                for (int e = 0; e < 9; ++e) fg_cgauss(seed, g, (uint32_t)k, (uint32_t)e, &m[2 * e], &m[2 * e + 1]);
            }
            if (scale != 1.0)
                for (int e = 0; e < 18; ++e) m[e] *= scale;
        }
    }
    return nloc * nper;
}

/* Full-box colour vector: out[local lex][3] complex. */
FG_API int64_t fg_vector(const int32_t G[4], const int32_t O[4], const int32_t E[4], uint64_t seed, double* out) {
    if (fg_check_box(G, O, E) || !out) return -1;
    const int64_t nloc = (int64_t)E[0] * E[1] * E[2] * E[3];
#pragma omp parallel for schedule(static)
    for (int64_t l = 0; l < nloc; ++l) {
        int64_t r = l;
        const int64_t x = r % E[0]; r /= E[0];
        const int64_t y = r % E[1]; r /= E[1];
        const int64_t z = r % E[2]; r /= E[2];
        const int64_t t = r;
        const uint64_t g = fg_glex(G, O[0] + x, O[1] + y, O[2] + z, O[3] + t);
        for (int c = 0; c < 3; ++c) fg_cgauss(seed, g, 0u, (uint32_t)c, &out[6 * l + 2 * c], &out[6 * l + 2 * c + 1]);
    }
    return nloc;
}

/*
 * The same vector values, but only the sites of GLOBAL parity `parity`, in the
 * library's checkerboard vector layout: out[c][cb] complex, c < 3, where
 * cb = (local lex) / 2 over the sites of that parity.  Requires E[0] even (then every
 * x-row holds E[0]/2 sites of each parity and cb is a bijection onto [0, Vh)), any
 * origin (odd origins describe ghost slabs).  Vh = nloc/2.
 */
FG_API int64_t fg_vector_cb(const int32_t G[4], const int32_t O[4], const int32_t E[4], uint64_t seed,
                            int32_t parity, double* out) {
    if (fg_check_box(G, O, E) || !out || (parity & ~1) || (E[0] & 1)) return -1;
    const int64_t osum = (int64_t)O[0] + O[1] + O[2] + O[3];
    const int64_t nloc = (int64_t)E[0] * E[1] * E[2] * E[3];
    const int64_t vh = nloc / 2;
#pragma omp parallel for schedule(static)
    for (int64_t l = 0; l < nloc; ++l) {
        int64_t r = l;
        const int64_t x = r % E[0]; r /= E[0];
        const int64_t y = r % E[1]; r /= E[1];
        const int64_t z = r % E[2]; r /= E[2];
        const int64_t t = r;
        if (((x + y + z + t + osum) & 1) != parity) continue;
        const uint64_t g = fg_glex(G, O[0] + x, O[1] + y, O[2] + z, O[3] + t);
        const int64_t cb = l >> 1;
        for (int c = 0; c < 3; ++c)
            fg_cgauss(seed, g, 0u, (uint32_t)c, &out[2 * (c * vh + cb)], &out[2 * (c * vh + cb) + 1]);
    }
    return vh;
}
