// l2_bw.cu -- L2-hit read bandwidth of the SMs (measurement aid for the 8-RHS analysis,
// profiles/r03/mrhs/): every thread reads 16-byte words of a buffer of `mb` MiB (resident in L2
// after the first pass) `reps` times, grid-stride, with ld.global.nc.L1::no_allocate; reports
// GB/s of bytes delivered to the SMs.  nvcc -gencode arch=compute_100a,code=sm_100a -O3 l2_bw.cu
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

__global__ void rd(const double2* __restrict__ p, size_t n, int reps, double* out, int inflight) {
    double acc = 0;
    const size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x, nt = (size_t)gridDim.x * blockDim.x;
    for (int r = 0; r < reps; ++r) {
        // offset the start per rep so a thread does not reread its own lines
        size_t i = (tid + (size_t)r * 977 * 32) % n;
        for (size_t k = 0; k + 8 <= n / nt; k += 8) {
            double2 v[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) {
                size_t j = i + (k + u) * nt;
                if (j >= n) j -= n;
                asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0, %1}, [%2];" : "=d"(v[u].x), "=d"(v[u].y) : "l"(p + j));
            }
#pragma unroll
            for (int u = 0; u < 8; ++u) acc += v[u].x + v[u].y;
        }
    }
    if (acc == 1.2345) out[0] = acc;
}

int main(int argc, char** argv) {
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    double* out;
    cudaMalloc(&out, 8);
    printf("mib blocks_per_sm threads GB/s\n");
    for (int mb : {16, 48, 96, 1024}) {
        size_t n = (size_t)mb * (1 << 20) / 16;
        double2* p;
        cudaMalloc(&p, n * 16);
        cudaMemset(p, 0, n * 16);
        for (int bps : {2, 4, 8}) {
            int threads = 256;
            int grid = sms * bps;
            int reps = mb >= 1024 ? 2 : 8;
            rd<<<grid, threads>>>(p, n, 1, out, 0);
            cudaEvent_t a, b;
            cudaEventCreate(&a);
            cudaEventCreate(&b);
            cudaEventRecord(a);
            rd<<<grid, threads>>>(p, n, reps, out, 0);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            if (cudaGetLastError() != cudaSuccess) { printf("kernel error\n"); return 1; }
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            size_t per_thread = (n / ((size_t)grid * threads)) / 8 * 8;
            double bytes = (double)per_thread * grid * threads * 16 * reps;
            printf("%5d %3d %4d %8.1f\n", mb, bps, threads, bytes / (ms * 1e-3) / 1e9); fflush(stdout);
        }
        cudaFree(p);
    }
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
