// Launch cost of a k_persist-shaped cooperative kernel (148 CTAs x 1024 threads, ~105 KB of
// dynamic shared memory, one grid barrier) as bench.py times it: an L2-flush write just before,
// CUDA events around the launch.  Variants separate the carve-out switch, the cooperative launch
// and the host submission.
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/microbench_coop.cu -o /tmp/mbc && /tmp/mbc
#include <cuda_runtime.h>
#include <stdio.h>

__device__ unsigned g_bar;
__device__ unsigned long long g_t[4];

__device__ __forceinline__ unsigned long long gt() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__global__ void k_fill(uint4* p, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
        p[i] = make_uint4(1, 1, 1, 1);
    if (blockIdx.x == 0 && threadIdx.x == 0) g_t[0] = gt();
}

__global__ __launch_bounds__(1024, 1) void k_coop(unsigned epoch) {
    extern __shared__ int sm[];
    if (threadIdx.x == 0) {
        atomicMin(&g_t[1], gt());
        sm[0] = 1;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        atomicAdd(&g_bar, 1u);
        while ((int)(*(volatile unsigned*)&g_bar - epoch * gridDim.x) < 0) {}
    }
    __syncthreads();
    if (threadIdx.x == 0) atomicMax(&g_t[2], gt());
}

int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    const size_t fill_bytes = 512ull << 20;
    uint4* buf;
    cudaMalloc(&buf, fill_bytes);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaStream_t s;
    cudaStreamCreate(&s);
    unsigned epoch = 0;
    struct V { const char* name; int smem; bool coop; bool fill; bool sync_before; int grid = 0; int block = 1024; };
    V vs[] = {
        {"coop smem105K, fill, host sync before", 105 << 10, true, true, true},
        {"coop smem105K, fill, no host sync", 105 << 10, true, true, false},
        {"coop smem105K, no fill, no host sync", 105 << 10, true, false, false},
        {"coop smem16, fill, no host sync", 16, true, true, false},
        {"plain smem105K, fill, no host sync", 105 << 10, false, true, false},
        {"plain smem16, fill, no host sync", 16, false, true, false},
        {"plain 148x256 smem16", 16, false, true, false, 0, 256},
        {"plain 74x1024 smem16", 16, false, true, false, 74, 1024},
        {"plain 1x32 (no barrier work)", 16, false, true, false, 1, 32},
    };
    cudaFuncSetAttribute(k_coop, cudaFuncAttributeMaxDynamicSharedMemorySize, 110 << 10);
    for (const V& v : vs) {
        double tot = 0, entry = 0;
        const int it = 50;
        for (int i = 0; i < it + 3; ++i) {
            unsigned long long init[4] = {0, ~0ull, 0, 0};
            cudaMemcpyToSymbol(g_t, init, sizeof(init));
            if (v.fill) k_fill<<<nsm * 4, 512, 0, s>>>(buf, fill_bytes / 16);
            if (v.sync_before) cudaStreamSynchronize(s);
            const unsigned zero = 0;
            cudaMemcpyToSymbolAsync(g_bar, &zero, sizeof(zero), 0, cudaMemcpyHostToDevice, s);
            cudaEventRecord(e0, s);
            epoch = 1;
            void* args[] = {&epoch};
            const int gridn = v.grid ? v.grid : nsm;
            if (v.coop) cudaLaunchCooperativeKernel((void*)k_coop, gridn, v.block, args, v.smem, s);
            else k_coop<<<gridn, v.block, v.smem, s>>>(epoch);
            cudaEventRecord(e1, s);
            cudaStreamSynchronize(s);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            unsigned long long t[4];
            cudaMemcpyFromSymbol(t, g_t, sizeof(t));
            if (i >= 3) {
                tot += ms * 1e3;
                entry += v.fill ? (double)(t[1] - t[0]) * 1e-3 : 0;
            }
        }
        printf("%-42s event %.2f us   fill end -> first CTA %.2f us\n", v.name, tot / it, entry / it);
    }
    cudaError_t err = cudaGetLastError();
    printf("status %s\n", cudaGetErrorString(err));
    return 0;
}
