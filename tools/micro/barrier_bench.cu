// Grid-barrier latency: cooperative_groups grid.sync() vs a two-level counter
// barrier, in a persistent cooperative kernel (the k_rounds launch shape).
#include <cooperative_groups.h>
#include <cstdio>
namespace cg = cooperative_groups;

struct GridBar {
    unsigned count[64 * 32];
    unsigned root;
    unsigned pad[31];
    unsigned gen;
};

__device__ __forceinline__ unsigned ld_acquire(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void bar2(GridBar* gb, unsigned& gen, int ngroups) {
    __syncthreads();
    if (threadIdx.x == 0) {
        const int G = gridDim.x;
        const int grp = blockIdx.x % ngroups;
        const int gsize = G / ngroups + (grp < G % ngroups ? 1 : 0);
        __threadfence();
        const unsigned a = atomicAdd(&gb->count[grp * 32], 1u) + 1;
        if (a == (unsigned)gsize) {
            gb->count[grp * 32] = 0;
            __threadfence();
            const unsigned r = atomicAdd(&gb->root, 1u) + 1;
            if (r == (unsigned)ngroups) {
                gb->root = 0;
                __threadfence();
                atomicAdd(&gb->gen, 1u);
            }
        }
        while (ld_acquire(&gb->gen) == gen) {
        }
        ++gen;
        __threadfence();
    }
    __syncthreads();
}

__global__ void k_cg(int iters, unsigned long long* out) {
    cg::grid_group grid = cg::this_grid();
    unsigned long long t0 = clock64();
    for (int i = 0; i < iters; ++i) grid.sync();
    if (blockIdx.x == 0 && threadIdx.x == 0) *out = clock64() - t0;
}

__global__ void k_bar(int iters, GridBar* gb, int ngroups, unsigned long long* out) {
    __shared__ unsigned gen_s;
    if (threadIdx.x == 0) gen_s = ld_acquire(&gb->gen);
    __syncthreads();
    unsigned gen = gen_s;
    unsigned long long t0 = clock64();
    for (int i = 0; i < iters; ++i) bar2(gb, gen, ngroups);
    if (blockIdx.x == 0 && threadIdx.x == 0) *out = clock64() - t0;
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    GridBar* gb;
    unsigned long long* out;
    cudaMalloc(&gb, sizeof(GridBar));
    cudaMemset(gb, 0, sizeof(GridBar));
    cudaMalloc(&out, 8);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    int iters = 2000;
    for (int ctas_per_sm : {1, 2}) {
        int G = sms * ctas_per_sm;
        void* args[] = {&iters, &out};
        cudaLaunchCooperativeKernel((void*)k_cg, G, 512, args, 0, 0);
        cudaEventRecord(a);
        cudaLaunchCooperativeKernel((void*)k_cg, G, 512, args, 0, 0);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        printf("cg grid.sync   G=%d: %.3f us/barrier\n", G, 1000.0 * ms / iters);
        for (int ng : {1, 8, 16, 32}) {
            void* args2[] = {&iters, &gb, &ng, &out};
            cudaLaunchCooperativeKernel((void*)k_bar, G, 512, args2, 0, 0);
            cudaEventRecord(a);
            cudaLaunchCooperativeKernel((void*)k_bar, G, 512, args2, 0, 0);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
            printf("two-level G=%d groups=%2d: %.3f us/barrier  (%s)\n", G, ng, 1000.0 * ms / iters,
                   cudaGetErrorString(cudaGetLastError()));
        }
    }
    return 0;
}
