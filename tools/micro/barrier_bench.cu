// Microbenchmark: cost of the library's grid barrier and of dependent global-memory round trips.
#include <cstdio>
#include <cuda_runtime.h>
#include "common.cuh"
using namespace ag;

__global__ void __launch_bounds__(256, 4) bar_kernel(Ctl *ctl, int iters, unsigned nblocks, unsigned long long *out) {
    __shared__ unsigned slot;
    unsigned gen = (unsigned)(ld_acquire64(&ctl->bar_word) >> 32);
    unsigned long long t0 = globaltimer_ns();
    for (int i = 0; i < iters; ++i) grid_sync(ctl, nblocks, &slot, gen, []() -> uint32_t { return 1u; });
    unsigned long long t1 = globaltimer_ns();
    if (blockIdx.x == 0 && threadIdx.x == 0) out[0] = t1 - t0;
}

__global__ void chase_kernel(const unsigned *next, int steps, unsigned long long *out, unsigned *sink) {
    unsigned p = 0;
    unsigned long long t0 = clock64();
    for (int i = 0; i < steps; ++i) p = __ldcg(next + p);
    unsigned long long t1 = clock64();
    sink[0] = p;
    out[1] = (t1 - t0) / steps;
}

__global__ void atom_chase_kernel(unsigned *ctr, int steps, unsigned long long *out) {
    unsigned p = 0;
    unsigned long long t0 = clock64();
    for (int i = 0; i < steps; ++i) p = atomicAdd(ctr + (p & 1), 1u) & 0;
    unsigned long long t1 = clock64();
    out[2] = (t1 - t0) / steps + p;
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    Ctl *ctl;
    cudaMalloc(&ctl, sizeof(Ctl));
    cudaMemset(ctl, 0, sizeof(Ctl));
    unsigned long long *out;
    cudaMallocManaged(&out, 64);
    for (int per : {1, 2, 4}) {
        unsigned nb = sms * per;
        int iters = 2000;
        void *args[] = {&ctl, &iters, &nb, &out};
        cudaLaunchCooperativeKernel((void *)bar_kernel, dim3(nb), dim3(256), args, 0, 0);
        cudaDeviceSynchronize();
        printf("grid_sync: %u CTAs: %.3f us per barrier\n", nb, out[0] / 1e3 / iters);
    }
    // pointer chase in a 64 MB array (L2 hits after warm-up within 126 MB L2) and 1 GB (DRAM)
    for (size_t n : {(size_t)1 << 14, (size_t)1 << 24, (size_t)1 << 28}) {
        unsigned *next, *sink;
        cudaMalloc(&next, n * 4);
        cudaMalloc(&sink, 4);
        unsigned *h = (unsigned *)malloc(n * 4);
        unsigned long long x = 1;
        for (size_t i = 0; i < n; ++i) { x = x * 6364136223846793005ull + 1442695040888963407ull; h[i] = (unsigned)((x >> 20) % n); }
        cudaMemcpy(next, h, n * 4, cudaMemcpyHostToDevice);
        chase_kernel<<<1, 1>>>(next, 1000, out, sink);
        chase_kernel<<<1, 1>>>(next, 10000, out, sink);
        cudaDeviceSynchronize();
        printf("dependent ld.cg chain, %zu MB: %llu cycles per load\n", n * 4 >> 20, out[1]);
        cudaFree(next); free(h);
    }
    unsigned *ctr;
    cudaMalloc(&ctr, 64);
    atom_chase_kernel<<<1, 1>>>(ctr, 10000, out);
    cudaDeviceSynchronize();
    printf("dependent atomicAdd chain: %llu cycles per atomic\n", out[2]);
    int clk;
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    printf("clock rate attr %d kHz; err=%s\n", clk, cudaGetErrorString(cudaGetLastError()));
    return 0;
}
