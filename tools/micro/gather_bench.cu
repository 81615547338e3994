// gather_bench.cu — throughput of random 4-byte status gathers on B200: L1/L2 (global) vs shared memory.
//
// The BFS/SSSP expansion issues one random status read per inspected edge.  This measures how many such
// reads per second the chip sustains from (a) a global table that fits L1 / L2, uniform or skewed index
// distribution, and (b) a shared-memory table, to decide where the status of the hot vertices lives.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gather_bench gather_bench.cu && ./gather_bench
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352du; x ^= x >> 15; x *= 0x846ca68bu; x ^= x >> 16;
    return x;
}
// skew: idx = N * u^3 (u uniform in [0,1)) concentrates on low ids like the degree layout
__device__ __forceinline__ uint32_t pick(uint32_t h, uint32_t n, int skew) {
    if (!skew) return h % n;
    const float u = (h >> 8) * (1.0f / 16777216.0f);
    return (uint32_t)(u * u * u * n);
}

template <int UNROLL>
__global__ void __launch_bounds__(256) gather_global(const uint32_t *tab, uint32_t n, int iters, int skew, uint32_t *sink) {
    uint32_t acc = 0;
    const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    for (int it = 0; it < iters; ++it) {
        uint32_t v[UNROLL];
#pragma unroll
        for (int j = 0; j < UNROLL; ++j) v[j] = __ldg(tab + pick(hash32(tid * 7919u + it * UNROLL + j), n, skew));
#pragma unroll
        for (int j = 0; j < UNROLL; ++j) acc += v[j];
    }
    if (acc == 0x12345678u) *sink = acc;
}

template <int UNROLL>
__global__ void __launch_bounds__(256) gather_global_plain(const uint32_t *tab, uint32_t n, int iters, int skew, uint32_t *sink) {
    uint32_t acc = 0;
    const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    for (int it = 0; it < iters; ++it) {
        uint32_t v[UNROLL];
#pragma unroll
        for (int j = 0; j < UNROLL; ++j) {
            const uint32_t *p = tab + pick(hash32(tid * 7919u + it * UNROLL + j), n, skew);
            asm volatile("ld.global.u32 %0, [%1];" : "=r"(v[j]) : "l"(p));
        }
#pragma unroll
        for (int j = 0; j < UNROLL; ++j) acc += v[j];
    }
    if (acc == 0x12345678u) *sink = acc;
}

template <int UNROLL>
__global__ void __launch_bounds__(1024) gather_smem(const uint32_t *tab, uint32_t n, int iters, int skew, uint32_t *sink) {
    extern __shared__ uint32_t s[];
    for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) s[i] = tab[i];
    __syncthreads();
    uint32_t acc = 0;
    const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    for (int it = 0; it < iters; ++it) {
        uint32_t v[UNROLL];
#pragma unroll
        for (int j = 0; j < UNROLL; ++j) v[j] = s[pick(hash32(tid * 7919u + it * UNROLL + j), n, skew)];
#pragma unroll
        for (int j = 0; j < UNROLL; ++j) acc += v[j];
    }
    if (acc == 0x12345678u) *sink = acc;
}

// ALU-only baseline: the index computation alone
template <int UNROLL>
__global__ void __launch_bounds__(256) alu_only(uint32_t n, int iters, int skew, uint32_t *sink) {
    uint32_t acc = 0;
    const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int j = 0; j < UNROLL; ++j) acc += pick(hash32(tid * 7919u + it * UNROLL + j), n, skew);
    }
    if (acc == 0x12345678u) *sink = acc;
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const uint32_t NMAX = 1u << 24;
    uint32_t *tab, *sink;
    cudaMalloc(&tab, NMAX * 4);
    cudaMalloc(&sink, 4);
    cudaMemset(tab, 1, NMAX * 4);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const int iters = 256;
    auto run = [&](const char *name, auto launch, double loads) {
        launch();
        cudaDeviceSynchronize();
        cudaEventRecord(a);
        for (int r = 0; r < 5; ++r) launch();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        ms /= 5;
        printf("%-52s %8.3f ms  %8.1f G loads/s  %6.2f loads/cyc/SM (1.965 GHz)\n", name, ms, loads / ms / 1e6,
               loads / (ms * 1e-3) / (sms * 1.965e9));
    };
    cudaError_t e = cudaFuncSetAttribute(gather_smem<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    if (e != cudaSuccess) printf("smem attr: %s\n", cudaGetErrorString(e));
    for (int skew = 0; skew < 2; ++skew) {
        const int grid = sms * 8;
        const double loads = (double)grid * 256 * iters * 8;
        char nm[128];
        snprintf(nm, sizeof nm, "alu only skew=%d", skew);
        run(nm, [&] { alu_only<8><<<grid, 256>>>(1u << 17, iters, skew, sink); }, loads);
        for (uint32_t n : {1u << 12, 1u << 14, 1u << 15, 1u << 17, 1u << 20, 1u << 22, 1u << 24}) {
            snprintf(nm, sizeof nm, "global ldg   n=%8u (%6u KB) skew=%d", n, n / 256, skew);
            run(nm, [&] { gather_global<8><<<grid, 256>>>(tab, n, iters, skew, sink); }, loads);
            snprintf(nm, sizeof nm, "global ld    n=%8u (%6u KB) skew=%d", n, n / 256, skew);
            run(nm, [&] { gather_global_plain<8><<<grid, 256>>>(tab, n, iters, skew, sink); }, loads);
        }
        for (uint32_t n : {1u << 12, 1u << 14, 1u << 15, 48u << 10}) {
            const int g2 = sms;
            const double l2 = (double)g2 * 1024 * iters * 8;
            snprintf(nm, sizeof nm, "smem         n=%8u (%6u KB) skew=%d", n, n / 256, skew);
            run(nm, [&] { gather_smem<8><<<g2, 1024, n * 4>>>(tab, n, iters, skew, sink); }, l2);
        }
    }
    e = cudaGetLastError();
    printf("last error: %s\n", cudaGetErrorString(e));
    return 0;
}
