// Does a scattered 4-byte store cost a DRAM read (sector read-modify-write) on B200?
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/microbench_scatter.cu -o /tmp/mbs
// ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum /tmp/mbs
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ unsigned long long mix(unsigned long long x) {
    x += 0x9e3779b97f4a7c15ull; x = (x ^ (x >> 30)) * 0xbf58476d1ce4e5b9ull;
    x = (x ^ (x >> 27)) * 0x94d049bb133111ebull; return x ^ (x >> 31);
}
__global__ void k_scatter(int* a, long long n, long long writes) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < writes; i += (long long)gridDim.x * blockDim.x)
        a[mix(i) % n] = (int)i;
}
__global__ void k_scatter_sector(int4* a, long long nsec, long long writes) {   // full 32-B sectors
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < writes; i += (long long)gridDim.x * blockDim.x) {
        long long s = mix(i) % nsec;
        a[2 * s] = make_int4(1, 2, 3, 4); a[2 * s + 1] = make_int4(5, 6, 7, 8);
    }
}
__global__ void k_fill(int4* a, long long n4) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n4; i += (long long)gridDim.x * blockDim.x)
        a[i] = make_int4(-1, -1, -1, -1);
}
int main() {
    const long long n = 1ll << 28;   // 1 GiB of int
    int* a; cudaMalloc(&a, n * 4);
    float ms;
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int rep = 0; rep < 2; ++rep) {
        k_fill<<<148 * 8, 256>>>((int4*)a, n / 4);
        cudaEventRecord(e0); k_fill<<<148 * 8, 256>>>((int4*)a, n / 4); cudaEventRecord(e1);
        cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
        printf("fill 1GiB: %.3f ms  %.1f GB/s\n", ms, n * 4 / ms / 1e6);
        const long long w = 1ll << 24;
        cudaEventRecord(e0); k_scatter<<<148 * 8, 256>>>(a, n, w); cudaEventRecord(e1);
        cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
        printf("scatter 16M x 4B into 1GiB: %.3f ms  %.1f Mwrites/s\n", ms, w / ms / 1e3);
        cudaEventRecord(e0); k_scatter_sector<<<148 * 8, 256>>>((int4*)a, n / 8, w); cudaEventRecord(e1);
        cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
        printf("scatter 16M x 32B sectors: %.3f ms  %.1f Mwrites/s\n", ms, w / ms / 1e3);
    }
    return 0;
}
