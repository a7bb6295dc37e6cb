// Launch-overhead microbenchmark for the per-level fixed cost (B200).
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/microbench_launch.cu -o /tmp/mb && /tmp/mb
#include <cuda_runtime.h>
#include <stdio.h>

__global__ void k_empty(int* p) {
    if (threadIdx.x == 0 && blockIdx.x == 0 && p) p[0]++;
}
__global__ void k_host_write(volatile int* h) {
    if (threadIdx.x == 0) h[0] = h[0] + 1;
}
__global__ __launch_bounds__(512) void k_smem41(int* p, int n) {
    __shared__ long long s[2049 * 2];
    __shared__ int si[2049];
    if (threadIdx.x < 4) { s[threadIdx.x] = threadIdx.x; si[threadIdx.x] = 1; }
    __syncthreads();
    if (blockIdx.x < n && threadIdx.x == 0) p[blockIdx.x] += (int)s[1] + si[0];
}
__global__ __launch_bounds__(256) void k_smem25(int* p) {
    __shared__ int s[6200];
    s[threadIdx.x] = threadIdx.x;
    __syncthreads();
    if (threadIdx.x == 0 && blockIdx.x == 0) p[1] += s[3];
}

template <class F>
float timeit(F f, int iters) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    for (int i = 0; i < 10; ++i) f();
    cudaEventRecord(a);
    for (int i = 0; i < iters; ++i) f();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    return ms * 1000.f / iters;
}

int main() {
    int* d;
    cudaMalloc(&d, 1 << 20);
    int* h;
    cudaHostAlloc(&h, 64, cudaHostAllocMapped);
    int* hd;
    cudaHostGetDevicePointer(&hd, h, 0);
    const int N = 2000;
    printf("empty 1x1              %.2f us/launch\n", timeit([&] { k_empty<<<1, 1>>>(d); }, N));
    printf("empty 592x512          %.2f us/launch\n", timeit([&] { k_empty<<<592, 512>>>(d); }, N));
    printf("host-mapped write 1x1  %.2f us/launch\n", timeit([&] { k_host_write<<<1, 1>>>(hd); }, N));
    printf("smem41 592x512         %.2f us/launch\n", timeit([&] { k_smem41<<<592, 512>>>(d, 8); }, N));
    printf("smem41 + empty         %.2f us/pair\n", timeit([&] { k_smem41<<<592, 512>>>(d, 8); k_empty<<<1, 1>>>(d); }, N));
    printf("smem41 + hostwrite     %.2f us/pair\n", timeit([&] { k_smem41<<<592, 512>>>(d, 8); k_host_write<<<1, 1>>>(hd); }, N));
    printf("smem41 + smem25        %.2f us/pair\n", timeit([&] { k_smem41<<<592, 512>>>(d, 8); k_smem25<<<1184, 256>>>(d); }, N));
    cudaFuncSetAttribute(k_smem41, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    cudaFuncSetAttribute(k_empty, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    cudaFuncSetAttribute(k_host_write, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    cudaFuncSetAttribute(k_smem25, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    printf("[carveout=100] smem41 + empty      %.2f us/pair\n", timeit([&] { k_smem41<<<592, 512>>>(d, 8); k_empty<<<1, 1>>>(d); }, N));
    printf("[carveout=100] smem41 + hostwrite  %.2f us/pair\n", timeit([&] { k_smem41<<<592, 512>>>(d, 8); k_host_write<<<1, 1>>>(hd); }, N));
    printf("[carveout=100] smem41 + smem25     %.2f us/pair\n", timeit([&] { k_smem41<<<592, 512>>>(d, 8); k_smem25<<<1184, 256>>>(d); }, N));
    // host-loop round trip: launch + sync
    printf("launch+sync empty      %.2f us\n", timeit([&] { k_empty<<<1, 1>>>(d); cudaStreamSynchronize(0); }, 500));
    printf("launch+sync hostwrite  %.2f us\n", timeit([&] { k_host_write<<<1, 1>>>(hd); cudaStreamSynchronize(0); }, 500));
    return 0;
}
