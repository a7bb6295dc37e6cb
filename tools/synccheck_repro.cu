// Minimal repro for the compute-sanitizer synccheck report on the CUDA-graph
// driver: a kernel whose __syncthreads sit in a
// block-uniform loop, launched (a) directly and (b) as a node inside a WHILE
// conditional graph node (the shape of libxbfs's device loop).  The kernel has
// no divergent barrier by construction: every thread of a block runs the same
// loop trip count.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/repro tools/synccheck_repro.cu
//   compute-sanitizer --tool synccheck /tmp/repro direct
//   compute-sanitizer --tool synccheck /tmp/repro graph
#include <cuda_runtime.h>
#include <stdio.h>
#include <string.h>

__global__ void k_body(const int* n, int* out) {
    __shared__ int s[512];
    const int trips = *n;                       // the same value for every thread
    for (int t = blockIdx.x; t < trips; t += gridDim.x) {
        __syncthreads();
        for (int i = threadIdx.x; i < 300; i += blockDim.x) s[i] = i + t;   // divergent tail, then converges
        __syncthreads();
        if (threadIdx.x == 0) atomicAdd(out, s[t % 300]);
    }
}

__global__ void k_step(cudaGraphConditionalHandle h, int* iter) {
    const int it = ++*iter;
    cudaGraphSetConditional(h, it < 3 ? 1u : 0u);
}

#define CK(x)                                                                        \
    do {                                                                             \
        cudaError_t e = (x);                                                         \
        if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return 1; } \
    } while (0)

int main(int argc, char** argv) {
    const bool graph = argc > 1 && !strcmp(argv[1], "graph");
    int *n, *out, *iter;
    CK(cudaMalloc(&n, sizeof(int)));
    CK(cudaMalloc(&out, sizeof(int)));
    CK(cudaMalloc(&iter, sizeof(int)));
    const int trips = 1000;
    CK(cudaMemcpy(n, &trips, sizeof(int), cudaMemcpyHostToDevice));
    CK(cudaMemset(out, 0, sizeof(int)));
    CK(cudaMemset(iter, 0, sizeof(int)));
    if (!graph) {
        for (int i = 0; i < 3; ++i) k_body<<<296, 512>>>(n, out);
        CK(cudaDeviceSynchronize());
    } else {
        cudaGraph_t g;
        CK(cudaGraphCreate(&g, 0));
        cudaGraphConditionalHandle h;
        CK(cudaGraphConditionalHandleCreate(&h, g, 1, cudaGraphCondAssignDefault));
        cudaGraphNodeParams wp = {};
        wp.type = cudaGraphNodeTypeConditional;
        wp.conditional.handle = h;
        wp.conditional.type = cudaGraphCondTypeWhile;
        wp.conditional.size = 1;
        cudaGraphNode_t wn, b0, b1;
        CK(cudaGraphAddNode(&wn, g, nullptr, 0, &wp));
        cudaGraph_t body = wp.conditional.phGraph_out[0];
        void* a0[] = {&n, &out};
        cudaKernelNodeParams p0 = {};
        p0.func = (void*)k_body;
        p0.gridDim = dim3(296);
        p0.blockDim = dim3(512);
        p0.kernelParams = a0;
        CK(cudaGraphAddKernelNode(&b0, body, nullptr, 0, &p0));
        void* a1[] = {&h, &iter};
        cudaKernelNodeParams p1 = {};
        p1.func = (void*)k_step;
        p1.gridDim = dim3(1);
        p1.blockDim = dim3(1);
        p1.kernelParams = a1;
        CK(cudaGraphAddKernelNode(&b1, body, &b0, 1, &p1));
        cudaGraphExec_t ex;
        CK(cudaGraphInstantiate(&ex, g, 0));
        CK(cudaGraphLaunch(ex, 0));
        CK(cudaDeviceSynchronize());
    }
    int h_out = 0;
    CK(cudaMemcpy(&h_out, out, sizeof(int), cudaMemcpyDeviceToHost));
    printf("%s ok: %d\n", graph ? "graph" : "direct", h_out);
    return 0;
}
