// stream_peak.cu -- achievable HBM bandwidth on this B200 for the access mixes the Dslash sees.
//
// The roofline denominator the bench reports is MEASURED_PEAKS.json's copy burst (read + write
// 1:1, torch copy_).  The Dslash moves 2352 B read per 48 B written, so a pure
// copy understates what HBM3e delivers to it.  This tool measures, with CUDA events over
// repeated launches on buffers far larger than L2:
//   read   : every byte read once (ld.global.nc.L1::no_allocate, 16 B per load), no writes;
//   mix48  : 48 bytes read per byte written (the Dslash ratio), reads as above, st.global.cs;
//   copy   : 1 byte read per byte written (the MEASURED_PEAKS convention).
// Grid = k x 148 SMs, grid-stride loops with UNROLL independent 16-byte loads in flight.
// Usage: stream_peak [GB]   (default 1.2 GB read per launch, the 32^4 link stream)
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x)                                                                           \
    do {                                                                                \
        cudaError_t e_ = (x);                                                           \
        if (e_ != cudaSuccess) {                                                        \
            fprintf(stderr, "%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e_)); \
            exit(1);                                                                    \
        }                                                                               \
    } while (0)

__device__ __forceinline__ double2 ld_nc(const double2* p) {
    double2 v;
    asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
    return v;
}

__device__ __forceinline__ void st_cs(double2* p, double2 v) {
    asm volatile("st.global.cs.v2.f64 [%0], {%1, %2};" ::"l"(p), "d"(v.x), "d"(v.y) : "memory");
}

// RATIO = 0: read only; otherwise one 16-byte store per RATIO 16-byte loads
template <int UNROLL, int RATIO>
__global__ void __launch_bounds__(256) stream_kernel(const double2* __restrict__ in, double2* __restrict__ out,
                                                     long long n, double* sink) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    double ax = 0, ay = 0;
    for (long long base = (long long)blockIdx.x * blockDim.x + threadIdx.x; base < n; base += stride * UNROLL) {
        double2 v[UNROLL];
#pragma unroll
        for (int u = 0; u < UNROLL; ++u) {
            const long long i = base + u * stride;
            v[u] = i < n ? ld_nc(in + i) : make_double2(0, 0);
        }
#pragma unroll
        for (int u = 0; u < UNROLL; ++u) {
            ax += v[u].x;
            ay += v[u].y;
            if constexpr (RATIO > 0) {
                const long long i = base + u * stride;
                if (i < n && ((unsigned)i % RATIO) == 0) st_cs(out + (unsigned)i / RATIO, v[u]);
            }
        }
    }
    if (ax == 1234.5 && ay == -1.0) *sink = ax;  // never true: keeps the loads alive
}

template <int UNROLL, int RATIO>
static double run(const double2* in, double2* out, long long n, double* sink, int blocks, int reps) {
    cudaEvent_t a, b;
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
    for (int w = 0; w < 3; ++w) stream_kernel<UNROLL, RATIO><<<blocks, 256>>>(in, out, n, sink);
    CK(cudaGetLastError());
    CK(cudaEventRecord(a));
    for (int r = 0; r < reps; ++r) stream_kernel<UNROLL, RATIO><<<blocks, 256>>>(in, out, n, sink);
    CK(cudaEventRecord(b));
    CK(cudaEventSynchronize(b));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, a, b));
    const double bytes = 16.0 * n * (1.0 + (RATIO > 0 ? 1.0 / RATIO : 0.0));
    return bytes * reps / (ms * 1e-3) / 1e9;
}

int main(int argc, char** argv) {
    const double gb = argc > 1 ? atof(argv[1]) : 1.2;
    const long long n = (long long)(gb * 1e9 / 16);
    double2 *in, *out;
    double* sink;
    CK(cudaMalloc(&in, n * sizeof(double2)));
    CK(cudaMalloc(&out, n * sizeof(double2)));
    CK(cudaMalloc(&sink, sizeof(double)));
    CK(cudaMemset(in, 0, n * sizeof(double2)));
    CK(cudaMemset(out, 0, n * sizeof(double2)));
    int sms = 0;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    const int reps = 50;
    double best_r = 0, best_m = 0, best_c = 0;
    for (int k : {4, 8, 16, 32}) {
        const int blocks = k * sms;
        const double r4 = run<4, 0>(in, out, n, sink, blocks, reps);
        const double r8 = run<8, 0>(in, out, n, sink, blocks, reps);
        const double m8 = run<8, 48>(in, out, n, sink, blocks, reps);
        const double c4 = run<4, 1>(in, out, n / 2, sink, blocks, reps);
        printf("blocks %5d: read %.1f / %.1f GB/s  mix48 %.1f GB/s  copy %.1f GB/s\n", blocks, r4, r8, m8, c4);
        best_r = std::max(best_r, std::max(r4, r8));
        best_m = std::max(best_m, m8);
        best_c = std::max(best_c, c4);
    }
    printf("{\"read_gbs\": %.1f, \"mix48_gbs\": %.1f, \"copy_gbs\": %.1f, \"bytes_read_per_launch\": %lld, "
           "\"sms\": %d}\n", best_r, best_m, best_c, 16 * n, sms);
    return 0;
}
