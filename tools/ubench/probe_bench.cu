// Microbenchmark: random 4-byte probes into a bitmap-sized array (B200).
// Measures probes/s for ld.global (default), ld.global.nc (__ldg), ld.global.cg,
// red.global.or, and shared-memory random loads, with 8 independent probes per
// thread in flight.  Used to size the visit step (a6) of the expand kernel.
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352d; x ^= x >> 15; x *= 0x846ca68b; x ^= x >> 16; return x;
}

template <int MODE>
__global__ void probe(const uint32_t* __restrict__ a, uint32_t* b, uint32_t nwords, uint32_t iters, uint32_t* out, uint32_t span_mask)
{
    __shared__ uint32_t sm[8192];  // 32 KB
    uint32_t acc = 0;
    uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    if (MODE == 4) { for (int i = threadIdx.x; i < 8192; i += blockDim.x) sm[i] = i; __syncthreads(); }
    uint32_t s = hash32(tid * 7919u + 1);
    for (uint32_t it = 0; it < iters; ++it) {
        uint32_t idx[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) { s = hash32(s + u); idx[u] = (s & span_mask) % nwords; }
        uint32_t v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            if (MODE == 0) v[u] = b[idx[u]];
            else if (MODE == 1) v[u] = __ldg(a + idx[u]);
            else if (MODE == 2) v[u] = __ldcg(a + idx[u]);
            else if (MODE == 3) { atomicOr(b + idx[u], 1u << (u & 31)); v[u] = 0; }
            else v[u] = sm[idx[u] & 8191];
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) acc += v[u];
    }
    if (acc == 0x12345678) out[0] = acc;
}

int main(int argc, char **argv) {
    // default 16.7M bits = 2 MiB (RMAT-24 visited bitmap); argv[1] = bits (C3: 41652230)
    const uint32_t nwords = (argc > 1 ? (uint32_t)atoll(argv[1]) : (1u << 24)) / 32;
    uint32_t *a, *b, *out;
    cudaMalloc(&a, nwords * 4); cudaMalloc(&b, nwords * 4); cudaMalloc(&out, 4);
    cudaMemset(a, 0x55, nwords * 4); cudaMemset(b, 0, nwords * 4);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const char* names[] = {"ld.global", "ld.global.nc", "ld.global.cg", "red.global.or", "ld.shared"};
    for (int mode = 0; mode < 5; ++mode) {
        for (int threads : {128, 256}) {
            int blocks = sms * (2048 / threads);
            if (mode == 4) blocks = sms * 4;
            uint32_t iters = 64;
            cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
            for (int rep = 0; rep < 2; ++rep) {
                cudaEventRecord(e0);
                switch (mode) {
                case 0: probe<0><<<blocks, threads>>>(a, b, nwords, iters, out, 0xffffffffu); break;
                case 1: probe<1><<<blocks, threads>>>(a, b, nwords, iters, out, 0xffffffffu); break;
                case 2: probe<2><<<blocks, threads>>>(a, b, nwords, iters, out, 0xffffffffu); break;
                case 3: probe<3><<<blocks, threads>>>(a, b, nwords, iters, out, 0xffffffffu); break;
                case 4: probe<4><<<blocks, threads>>>(a, b, nwords, iters, out, 0xffffffffu); break;
                }
                cudaEventRecord(e1); cudaEventSynchronize(e1);
            }
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            double probes = (double)blocks * threads * iters * 8;
            printf("%-16s threads=%d blocks=%d : %.1f G probes/s (%.3f ms) err=%s\n", names[mode], threads, blocks,
                   probes / ms / 1e6, ms, cudaGetErrorString(cudaGetLastError()));
        }
    }
    return 0;
}
