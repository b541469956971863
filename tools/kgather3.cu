// kgather3.cu — is the random-miss ceiling SM-side or memory-side?
// Persistent CTAs (8 x 256 threads per SM, full occupancy) pull work from an atomic
// counter; CTAs on SMs >= active_sms exit at once, so only `active_sms` SMs load.
// Power-of-two buffer => mask instead of modulo (no 64-bit division on the path).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

__global__ void __launch_bounds__(256) gather(const uint8_t* __restrict__ buf, uint64_t mask, uint64_t n,
                                              unsigned long long* ctr, int active_sms, uint64_t* out) {
    uint32_t smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    if (smid >= (uint32_t)active_sms) return;
    __shared__ uint64_t chunk;
    uint64_t acc = 0;
    for (;;) {
        if (threadIdx.x == 0) chunk = atomicAdd(ctr, 256ull * 16);
        __syncthreads();
        const uint64_t c0 = chunk;
        __syncthreads();
        if (c0 >= n) break;
#pragma unroll 4
        for (int r = 0; r < 16; r++) {
            const uint64_t i = c0 + r * 256 + threadIdx.x;
            const uint64_t s = mix(i) & mask;
            uint64_t v;
            asm volatile("ld.global.nc.u64 %0, [%1];" : "=l"(v) : "l"(buf + s * 64));
            acc += v;
        }
    }
    if (acc == 0x1234567) out[0] = acc;
}

int main() {
    const size_t bytes = 8ull << 30;
    uint8_t* buf;
    uint64_t* out;
    unsigned long long* ctr;
    cudaMalloc(&buf, bytes);
    cudaMalloc(&out, 64);
    cudaMalloc(&ctr, 8);
    cudaMemset(buf, 1, bytes);
    const uint64_t mask = bytes / 64 - 1;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    for (int sms : {8, 16, 37, 74, 111, 148}) {
        const uint64_t n = uint64_t(sms) * 4000000ull;
        for (int rep = 0; rep < 2; rep++) {
            cudaMemset(ctr, 0, 8);
            cudaEventRecord(a);
            gather<<<148 * 8, 256>>>(buf, mask, n, ctr, sms, out);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
        }
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        printf("{\"active_sms\": %d, \"loads\": %llu, \"ms\": %.3f, \"Gloads_s\": %.2f, \"per_sm_Gloads_s\": %.3f}\n", sms,
               (unsigned long long)n, ms, n / (ms * 1e-3) / 1e9, n / (ms * 1e-3) / 1e9 / sms);
    }
    return 0;
}
