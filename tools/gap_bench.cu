// Per-iteration launch overhead of the iteration loop (calibration, not product code):
//  (a) CUDA-graph conditional WHILE node with two kernel nodes per body (the
//      fused loop's structure: expand 444 CTAs, scan 592 CTAs);
//  (b) the same two kernels launched back to back on a stream;
//  (c) one persistent kernel (444 CTAs) with two software grid barriers per iteration.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gap_bench tools/gap_bench.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); return 1; } } while (0)

struct Ctl { unsigned iter, N, bar_count, bar_gen, sink; };

__global__ void k_exp(Ctl *c) {
    if (threadIdx.x == 0 && c->iter == 0xFFFFFFFFu) c->sink = blockIdx.x;
}
__global__ void k_scan(Ctl *c, cudaGraphConditionalHandle h, int use) {
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        unsigned it = ++c->iter;
        if (use) cudaGraphSetConditional(h, it < c->N ? 1u : 0u);
    }
}

__device__ __forceinline__ void grid_barrier(Ctl *c, unsigned &gen) {
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        const unsigned g = gen;
        if (atomicAdd(&c->bar_count, 1u) == gridDim.x - 1) {
            c->bar_count = 0;
            __threadfence();
            atomicExch(&c->bar_gen, g + 1);
        } else {
            while (*(volatile unsigned *)&c->bar_gen == g) __nanosleep(32);
        }
        __threadfence();
    }
    ++gen;
    __syncthreads();
}

__global__ void k_persist(Ctl *c) {
    unsigned gen = *(volatile unsigned *)&c->bar_gen;
    for (unsigned it = 0; it < c->N; ++it) {
        if (threadIdx.x == 0 && c->iter == 0xFFFFFFFFu) c->sink = blockIdx.x;
        grid_barrier(c, gen);
        grid_barrier(c, gen);
    }
}

int main() {
    const unsigned N = 400;
    Ctl *c;
    CK(cudaMalloc(&c, sizeof(Ctl)));
    cudaStream_t s;
    CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    Ctl h = {0, N, 0, 0, 0};
    float ms;

    // (a) graph while loop
    cudaGraph_t graph;
    CK(cudaGraphCreate(&graph, 0));
    cudaGraphConditionalHandle cond;
    CK(cudaGraphConditionalHandleCreate(&cond, graph, 1, cudaGraphCondAssignDefault));
    cudaGraphNodeParams cp = {};
    cp.type = cudaGraphNodeTypeConditional;
    cp.conditional.handle = cond;
    cp.conditional.type = cudaGraphCondTypeWhile;
    cp.conditional.size = 1;
    cudaGraphNode_t cnode, n1, n2;
    CK(cudaGraphAddNode(&cnode, graph, nullptr, 0, &cp));
    cudaGraph_t body = cp.conditional.phGraph_out[0];
    cudaKernelNodeParams kp = {};
    void *a1[] = {&c};
    kp.func = (void *)k_exp; kp.gridDim = dim3(444); kp.blockDim = dim3(256); kp.kernelParams = a1;
    CK(cudaGraphAddKernelNode(&n1, body, nullptr, 0, &kp));
    int one = 1;
    void *a2[] = {&c, &cond, &one};
    kp.func = (void *)k_scan; kp.gridDim = dim3(592); kp.kernelParams = a2;
    CK(cudaGraphAddKernelNode(&n2, body, &n1, 1, &kp));
    cudaGraphExec_t exec;
    CK(cudaGraphInstantiate(&exec, graph, 0));
    for (int rep = 0; rep < 3; ++rep) {
        CK(cudaMemcpyAsync(c, &h, sizeof(h), cudaMemcpyHostToDevice, s));
        CK(cudaEventRecord(e0, s));
        CK(cudaGraphLaunch(exec, s));
        CK(cudaEventRecord(e1, s));
        CK(cudaStreamSynchronize(s));
        CK(cudaEventElapsedTime(&ms, e0, e1));
        printf("graph while: %.2f us / iteration\n", ms * 1000.f / N);
    }
    // (b) stream launches
    cudaGraphConditionalHandle none = 0;
    int zero = 0;
    for (int rep = 0; rep < 3; ++rep) {
        CK(cudaMemcpyAsync(c, &h, sizeof(h), cudaMemcpyHostToDevice, s));
        CK(cudaEventRecord(e0, s));
        for (unsigned i = 0; i < N; ++i) {
            k_exp<<<444, 256, 0, s>>>(c);
            k_scan<<<592, 256, 0, s>>>(c, none, zero);
        }
        CK(cudaEventRecord(e1, s));
        CK(cudaStreamSynchronize(s));
        CK(cudaEventElapsedTime(&ms, e0, e1));
        printf("stream launches: %.2f us / iteration\n", ms * 1000.f / N);
    }
    // (c) persistent kernel, two grid barriers per iteration
    for (int rep = 0; rep < 3; ++rep) {
        CK(cudaMemcpyAsync(c, &h, sizeof(h), cudaMemcpyHostToDevice, s));
        void *a3[] = {&c};
        CK(cudaEventRecord(e0, s));
        CK(cudaLaunchCooperativeKernel((void *)k_persist, dim3(444), dim3(256), a3, 0, s));
        CK(cudaEventRecord(e1, s));
        CK(cudaStreamSynchronize(s));
        CK(cudaEventElapsedTime(&ms, e0, e1));
        printf("persistent, 2 barriers: %.2f us / iteration\n", ms * 1000.f / N);
    }
    return 0;
}
