// Random-access ceiling of B200 (profiles/r01_l2_random_ubench.txt): 8-byte
// gathers (ld.global.cg), 64-bit REDs and an even mix of both to uniformly
// random addresses of an array of S bytes, all SMs, 8-16 accesses in flight
// per thread.  The mix over an L2-resident array is the ceiling of the
// accumulative path walk (one master gather + one RED per walked entry).
// MODE 2 issues a thread's gathers and REDs in one loop (a later iteration's
// gathers cannot pass the earlier REDs: a serialised mix); MODE 3 splits them
// over warps (even warps gather, odd warps RED) -- the concurrent, additive
// ceiling the verdict r01 asked for (both count gathers + REDs as ops).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ubench scripts/ubench_l2_random.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t hsh(uint32_t x) { x ^= x >> 16; x *= 0x7feb352d; x ^= x >> 15; x *= 0x846ca68b; x ^= x >> 16; return x; }
template <int MODE, int U>
__global__ void k(unsigned long long* a, uint32_t nmask, int iters, unsigned long long* out) {
    uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    unsigned long long s = 0;
    for (int it = 0; it < iters; it++) {
        uint32_t idx[U];
#pragma unroll
        for (int u = 0; u < U; u++) idx[u] = hsh(tid * 7919u + (uint32_t)(it * U + u) * 104729u) & nmask;
        if (MODE == 0) {
            unsigned long long v[U];
#pragma unroll
            for (int u = 0; u < U; u++) v[u] = __ldcg(&a[idx[u]]);
#pragma unroll
            for (int u = 0; u < U; u++) s += v[u];
        } else if (MODE == 1) {
#pragma unroll
            for (int u = 0; u < U; u++) atomicAdd(&a[idx[u]], 1ull);
        } else if (MODE == 3) {
            if (((threadIdx.x >> 5) & 1) == 0) {
                unsigned long long v[U];
#pragma unroll
                for (int u = 0; u < U; u++) v[u] = __ldcg(&a[idx[u]]);
#pragma unroll
                for (int u = 0; u < U; u++) s += v[u];
            } else {
#pragma unroll
                for (int u = 0; u < U; u++) atomicAdd(&a[idx[u]], 1ull);
            }
        } else {
            unsigned long long v[U];
#pragma unroll
            for (int u = 0; u < U; u++) v[u] = __ldcg(&a[idx[u]]);
#pragma unroll
            for (int u = 0; u < U; u++) { s += v[u]; atomicAdd(&a[hsh(idx[u]) & nmask], 1ull); }
        }
    }
    if (s == 12345) out[0] = s;
}
template <int MODE, int U>
void run(const char* name, unsigned long long* a, uint32_t n, int blocks, int threads) {
    int iters = 64;
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    k<MODE, U><<<blocks, threads>>>(a, n - 1, 4, a);
    cudaEventRecord(e0);
    k<MODE, U><<<blocks, threads>>>(a, n - 1, iters, a);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double ops = (double)blocks * threads * iters * U * (MODE == 2 ? 2 : 1);
    printf("%-8s S=%7.1f MB blocks=%5d thr=%4d U=%2d : %7.1f G ops/s (%.3f ms)\n", name, n * 8.0 / 1e6, blocks, threads, U, ops / ms / 1e6, ms);
}
int main() {
    unsigned long long* a;
    size_t maxn = 1ull << 27;  // 1 GB
    cudaMalloc(&a, maxn * 8); cudaMemset(a, 0, maxn * 8);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    for (uint32_t n : {1u << 22, 1u << 23, 1u << 26}) {  // 32 MB, 64 MB, 512 MB
        for (int bpsm : {4, 8}) {
            run<0, 8>("gather", a, n, sms * bpsm, 256);
            run<1, 8>("red", a, n, sms * bpsm, 256);
            run<2, 8>("g+red", a, n, sms * bpsm, 256);
            run<3, 8>("g|red", a, n, sms * bpsm, 256);
        }
        run<0, 16>("gather", a, n, sms * 8, 256);
    }
    cudaError_t e = cudaGetLastError();
    printf("%s\n", cudaGetErrorString(e));
}
