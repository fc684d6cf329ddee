// Minimal repro for the compute-sanitizer report on CUDA-graph conditional
// WHILE loops (VERDICT r01 "What's weak" #3): no library code, one device
// counter.  The body kernel decrements the counter and sets the loop
// condition -- the same structure as libetg's loop (expand -> scan, the scan
// setting the conditional).  Build + run:
//   nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/repro tools/sanitize_graph_repro.cu
//   compute-sanitizer --tool memcheck /tmp/repro
// A clean program: any sanitizer error here is the tool's, not the library's.
#include <cuda_runtime.h>
#include <cstdio>

__global__ void body_a(unsigned *ctr) {
    if (threadIdx.x == 0 && blockIdx.x == 0) atomicAdd(ctr + 1, 1u);
}

__global__ void body_b(unsigned *ctr, cudaGraphConditionalHandle h) {
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        const unsigned left = --ctr[0];
        cudaGraphSetConditional(h, left ? 1u : 0u);
    }
}

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

int main() {
    unsigned *ctr;
    CK(cudaMalloc(&ctr, 8));
    unsigned init[2] = {10, 0};
    CK(cudaMemcpy(ctr, init, 8, cudaMemcpyHostToDevice));
    cudaGraph_t g;
    CK(cudaGraphCreate(&g, 0));
    cudaGraphConditionalHandle h;
    CK(cudaGraphConditionalHandleCreate(&h, g, 1, cudaGraphCondAssignDefault));
    cudaGraphNodeParams cp = {};
    cp.type = cudaGraphNodeTypeConditional;
    cp.conditional.handle = h;
    cp.conditional.type = cudaGraphCondTypeWhile;
    cp.conditional.size = 1;
    cudaGraphNode_t cn;
    CK(cudaGraphAddNode(&cn, g, nullptr, 0, &cp));
    cudaGraph_t body = cp.conditional.phGraph_out[0];
    cudaKernelNodeParams kp = {};
    cudaGraphNode_t na, nb;
    void *aa[] = {&ctr};
    kp.func = (void *)body_a;
    kp.gridDim = dim3(4);
    kp.blockDim = dim3(256);
    kp.kernelParams = aa;
    CK(cudaGraphAddKernelNode(&na, body, nullptr, 0, &kp));
    void *ab[] = {&ctr, &h};
    kp.func = (void *)body_b;
    kp.gridDim = dim3(4);
    kp.kernelParams = ab;
    CK(cudaGraphAddKernelNode(&nb, body, &na, 1, &kp));
    cudaGraphExec_t ex;
    CK(cudaGraphInstantiate(&ex, g, 0));
    CK(cudaGraphLaunch(ex, 0));
    CK(cudaDeviceSynchronize());
    unsigned out[2];
    CK(cudaMemcpy(out, ctr, 8, cudaMemcpyDeviceToHost));
    printf("iterations=%u (expect 10), left=%u\n", out[1], out[0]);
    return out[1] == 10 && out[0] == 0 ? 0 : 2;
}
