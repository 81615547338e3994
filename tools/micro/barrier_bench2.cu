// Compare grid-barrier implementations (cost per barrier, us).
#include <cstdio>
#include <cuda_runtime.h>
#include <cooperative_groups.h>
#include "common.cuh"
using namespace ag;
namespace cg = cooperative_groups;

__device__ __forceinline__ unsigned atom_add_relaxed(unsigned *p, unsigned v) {
    unsigned old;
    asm volatile("atom.relaxed.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
    return old;
}
__device__ __forceinline__ void red_release(unsigned *p, unsigned v) {
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// V1: flat counter, threadfence + relaxed atomics
__device__ void bar_flat(Ctl *ctl, unsigned nb, unsigned &gen) {
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        if (atom_add_relaxed(&ctl->bar_count, 1u) == nb - 1) {
            ctl->bar_count = 0;
            __threadfence();
            st_release64(&ctl->bar_word, (unsigned long long)(gen + 1) << 32);
        }
        while ((unsigned)(ld_relaxed64(&ctl->bar_word) >> 32) == gen) {}
        __threadfence();
    }
    gen++;
    __syncthreads();
}
// V2: monotone counter (no reset): arrive with red.release, wait until count >= (gen+1)*nb
__device__ void bar_mono(Ctl *ctl, unsigned nb, unsigned &gen) {
    __syncthreads();
    if (threadIdx.x == 0) {
        red_release(&ctl->bar_count, 1u);
        const unsigned target = (gen + 1) * nb;
        while ((int)(ld_acquire(&ctl->bar_count) - target) < 0) {}
    }
    gen++;
    __syncthreads();
}
// V3: monotone counter, relaxed polling + final acquire
__device__ void bar_mono2(Ctl *ctl, unsigned nb, unsigned &gen) {
    __syncthreads();
    if (threadIdx.x == 0) {
        red_release(&ctl->bar_count, 1u);
        const unsigned target = (gen + 1) * nb;
        while ((int)(ld_relaxed(&ctl->bar_count) - target) < 0) {}
        (void)ld_acquire(&ctl->bar_count);
    }
    gen++;
    __syncthreads();
}

template <int V>
__global__ void __launch_bounds__(256, 4) bk(Ctl *ctl, int iters, unsigned nb, unsigned long long *out) {
    __shared__ unsigned slot;
    unsigned gen = 0;
    if (V == 0) gen = (unsigned)(ld_acquire64(&ctl->bar_word) >> 32);
    unsigned long long t0 = globaltimer_ns();
    for (int i = 0; i < iters; ++i) {
        if (V == 0) grid_sync(ctl, nb, &slot, gen, []() -> uint32_t { return 1u; });
        if (V == 1) bar_flat(ctl, nb, gen);
        if (V == 2) bar_mono(ctl, nb, gen);
        if (V == 3) bar_mono2(ctl, nb, gen);
        if (V == 4) cg::this_grid().sync();
    }
    unsigned long long t1 = globaltimer_ns();
    if (blockIdx.x == 0 && threadIdx.x == 0) out[0] = t1 - t0;
}

template <int V>
void run(const char *name, Ctl *ctl, unsigned long long *out, int sms) {
    for (int per : {1, 4, 8}) {
        cudaMemset(ctl, 0, sizeof(Ctl));
        unsigned nb = sms * per;
        int iters = 2000;
        void *args[] = {&ctl, &iters, &nb, &out};
        cudaError_t e = cudaLaunchCooperativeKernel((void *)bk<V>, dim3(nb), dim3(256), args, 0, 0);
        cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("%s %u: %s\n", name, nb, cudaGetErrorString(e)); continue; }
        printf("%-28s %4u CTAs: %.3f us/barrier\n", name, nb, out[0] / 1e3 / iters);
    }
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    Ctl *ctl;
    cudaMalloc(&ctl, sizeof(Ctl));
    unsigned long long *out;
    cudaMallocManaged(&out, 64);
    run<0>("hierarchical acq_rel", ctl, out, sms);
    run<1>("flat threadfence", ctl, out, sms);
    run<2>("monotone red.release/acq", ctl, out, sms);
    run<3>("monotone relaxed poll", ctl, out, sms);
    run<4>("cooperative_groups", ctl, out, sms);
    return 0;
}
