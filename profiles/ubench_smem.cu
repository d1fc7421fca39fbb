// Microbenchmark: shared-memory insert primitives on B200 (random addresses).
#include <cstdio>
#include <cuda_runtime.h>
#define N_ITERS 4096
template <int MODE>
__global__ void k(unsigned* out, unsigned seed) {
    extern __shared__ unsigned sm[];
    const unsigned words = 16384;  // 64 KB
    for (unsigned i = threadIdx.x; i < words; i += blockDim.x) sm[i] = 0xFFFFFFFFu * (MODE == 1);
    __syncthreads();
    unsigned x = seed ^ (threadIdx.x * 2654435761u) ^ (blockIdx.x * 97u);
    unsigned acc = 0;
    for (int i = 0; i < N_ITERS; ++i) {
        x = x * 1664525u + 1013904223u;
        unsigned w = (x >> 8) & (words - 1);
        if (MODE == 0) atomicOr(&sm[w], 1u << (x & 31));
        else if (MODE == 1) acc += atomicCAS(&sm[w], 0xFFFFFFFFu, x);
        else if (MODE == 2) ((unsigned char*)sm)[(x >> 6) & (words * 4 - 1)] = 1;
        else if (MODE == 3) sm[w] = x;
        else if (MODE == 4) acc += sm[w];
        else if (MODE == 5) atomicAdd(&sm[w], 1u);
        else if (MODE == 6) { if (sm[w] != x) atomicCAS(&sm[w], 0xFFFFFFFFu, x); }
    }
    __syncthreads();
    if (threadIdx.x == 0) out[blockIdx.x] = sm[7] + acc;
}
template <int MODE> void run(const char* name, int blocks_per_sm, int threads) {
    unsigned* out; cudaMalloc(&out, 148 * 64 * 4);
    cudaFuncSetAttribute(k<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
    int grid = 148 * blocks_per_sm;
    k<MODE><<<grid, threads, 65536>>>(out, 1);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a);
    k<MODE><<<grid, threads, 65536>>>(out, 2);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    double ops = double(grid) * threads * N_ITERS;
    printf("%-28s blocks/SM %d thr %4d : %8.2f Gops/s  (%.3f ms)  err=%s\n", name, blocks_per_sm, threads, ops / ms / 1e6, ms,
           cudaGetErrorString(cudaGetLastError()));
    cudaFree(out);
}
int main() {
    for (int t : {512, 1024}) for (int bps : {1, 3}) {
        if (t * bps > 2048) continue;
        run<0>("atomicOr smem", bps, t);
        run<1>("atomicCAS smem", bps, t);
        run<6>("load-check + CAS", bps, t);
        run<5>("atomicAdd smem", bps, t);
        run<2>("STS.U8 byte", bps, t);
        run<3>("STS.32", bps, t);
        run<4>("LDS.32", bps, t);
    }
}
