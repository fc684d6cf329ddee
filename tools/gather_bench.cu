// gather_bench.cu -- calibration microbenchmark (not part of the library):
// throughput of random 4-byte gathers / atomics on a label-sized array, the
// access pattern that bounds the expand kernel.  Build and run on the GPU box:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/gb tools/gather_bench.cu && /tmp/gb
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int R, int MODE>
__global__ void gather(const uint32_t *__restrict__ idx, uint32_t *lab, uint64_t n_idx, uint32_t *out) {
    uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    uint32_t acc = 0;
    for (uint64_t base = tid; base + (R - 1) * stride < n_idx; base += R * stride) {
        uint32_t u[R], v[R];
#pragma unroll
        for (int r = 0; r < R; ++r) u[r] = idx[base + r * stride];
#pragma unroll
        for (int r = 0; r < R; ++r) {
            if (MODE == 0) v[r] = __ldcg(&lab[u[r]]);
            else if (MODE == 1) asm volatile("ld.global.ca.u32 %0, [%1];" : "=r"(v[r]) : "l"(&lab[u[r]]));
            else if (MODE == 2) v[r] = __ldg(&lab[u[r]]);
            else if (MODE == 3) v[r] = atomicMin(&lab[u[r]], 7u);
            else { asm volatile("red.relaxed.gpu.global.min.u32 [%0], %1;" :: "l"(&lab[u[r]]), "r"(u[r] & 1023u) : "memory"); v[r] = 0; }
        }
#pragma unroll
        for (int r = 0; r < R; ++r) acc += v[r];
    }
    if (acc == 0x12345678) out[0] = acc;
}

__global__ void fill_idx(uint32_t *idx, uint64_t n_idx, uint32_t n, uint32_t seed) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n_idx; i += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t z = (i + seed) * 0x9E3779B97F4A7C15ull;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        z ^= z >> 31;
        idx[i] = (uint32_t)(z % n);
    }
}

template <int R, int MODE>
void run(const char *name, const uint32_t *idx, uint32_t *lab, uint64_t n_idx, uint32_t *out, int sms, int bps, int threads) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    gather<R, MODE><<<sms * bps, threads>>>(idx, lab, n_idx, out);
    cudaEventRecord(a);
    for (int k = 0; k < 5; ++k) gather<R, MODE><<<sms * bps, threads>>>(idx, lab, n_idx, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    printf("%-8s R=%2d blocks/SM=%2d threads=%4d : %7.1f G accesses/s\n", name, R, bps, threads,
           5.0 * n_idx / (ms * 1e-3) / 1e9);
}

int main(int argc, char **argv) {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const uint32_t n = 1u << 22;                 // C2 label array: 16.8 MB
    const uint64_t n_idx = 64ull << 20;          // 64M random targets
    uint32_t *idx, *lab, *out;
    cudaMalloc(&idx, n_idx * 4);
    cudaMalloc(&lab, (uint64_t)n * 4);
    cudaMalloc(&out, 4);
    cudaMemset(lab, 0xFF, (uint64_t)n * 4);
    fill_idx<<<sms * 8, 256>>>(idx, n_idx, n, 1);
    cudaDeviceSynchronize();
    if (argc > 1) {                 // index stream from a file of uint32 (e.g. the C2 col array)
        FILE *f = fopen(argv[1], "rb");
        uint32_t *h = (uint32_t *)malloc(n_idx * 4);
        size_t got = fread(h, 4, n_idx, f);
        fclose(f);
        printf("loaded %zu indices from %s\n", got, argv[1]);
        cudaMemcpy(idx, h, got * 4, cudaMemcpyHostToDevice);
        free(h);
    }
    for (int bps : {1, 2}) {
        run<8, 0>("ld.cg", idx, lab, n_idx, out, sms, bps, 256);
        run<16, 0>("ld.cg", idx, lab, n_idx, out, sms, bps, 256);
        run<32, 0>("ld.cg", idx, lab, n_idx, out, sms, bps, 256);
    }
    for (int bps : {4, 8}) {
        run<1, 0>("ld.cg", idx, lab, n_idx, out, sms, bps, 256);
        run<8, 0>("ld.cg", idx, lab, n_idx, out, sms, bps, 256);
        run<16, 0>("ld.cg", idx, lab, n_idx, out, sms, bps, 256);
        run<8, 1>("ld.ca", idx, lab, n_idx, out, sms, bps, 256);
        run<8, 2>("ld.nc", idx, lab, n_idx, out, sms, bps, 256);
        run<8, 3>("atomMin", idx, lab, n_idx, out, sms, bps, 256);
        run<8, 4>("redMin", idx, lab, n_idx, out, sms, bps, 256);
    }
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
