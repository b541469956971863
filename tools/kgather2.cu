// kgather2.cu — where does the ~47 G/s random-miss ceiling come from?
//  (a) SM-count scaling: same random 8-B gather on 37 / 74 / 148 SMs (1 CTA of 1024 threads per SM, forced by smem)
//  (b) the same gather through cp.async (LDGSTS, 16 B) and TMA bulk copies (cp.async.bulk, 16 B) into smem
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

__global__ void __launch_bounds__(1024) ldg(const uint8_t* __restrict__ buf, uint64_t slots, uint64_t n, uint64_t* out) {
    extern __shared__ uint8_t sm[];
    uint64_t acc = 0;
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n / 4; i += stride) {
        uint64_t v[4];
#pragma unroll
        for (int r = 0; r < 4; r++) {
            const uint64_t s = mix(i * 4 + r) % slots;
            asm volatile("ld.global.nc.u64 %0, [%1];" : "=l"(v[r]) : "l"(buf + s * 64));
        }
        acc += v[0] + v[1] + v[2] + v[3];
    }
    if (acc == 0x1234567) out[0] = acc + sm[0];
}

// cp.async 16 B per thread into its own smem slot, 4 in flight per thread
__global__ void __launch_bounds__(256) ldgsts(const uint8_t* __restrict__ buf, uint64_t slots, uint64_t n, uint64_t* out) {
    __shared__ __align__(16) uint8_t sm[256 * 4 * 16];
    uint64_t acc = 0;
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    uint32_t base = (uint32_t)__cvta_generic_to_shared(sm + threadIdx.x * 64);
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n / 4; i += stride) {
#pragma unroll
        for (int r = 0; r < 4; r++) {
            const uint64_t s = mix(i * 4 + r) % slots;
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(base + 16 * r), "l"(buf + s * 64));
        }
        asm volatile("cp.async.commit_group;");
        asm volatile("cp.async.wait_group 0;");
        acc += *(uint64_t*)(sm + threadIdx.x * 64) + *(uint64_t*)(sm + threadIdx.x * 64 + 48);
    }
    if (acc == 0x1234567) out[0] = acc;
}

// TMA bulk copy (non-tensor) 16 B per thread, one mbarrier per warp, 4 copies per lane in flight
__global__ void __launch_bounds__(256) bulk(const uint8_t* __restrict__ buf, uint64_t slots, uint64_t n, uint64_t* out) {
    __shared__ __align__(128) uint8_t sm[256 * 4 * 16];
    __shared__ __align__(8) uint64_t bar[8];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    uint32_t mb = (uint32_t)__cvta_generic_to_shared(&bar[warp]);
    if (lane == 0) asm volatile("mbarrier.init.shared.b64 [%0], 1;" :: "r"(mb));
    __syncwarp();
    asm volatile("fence.mbarrier_init.release.cluster;");
    __syncwarp();
    uint64_t acc = 0;
    uint32_t phase = 0;
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    uint32_t dst = (uint32_t)__cvta_generic_to_shared(sm + threadIdx.x * 64);
    const uint64_t iters = (n / 4 + stride - 1) / stride;
    for (uint64_t it = 0; it < iters; it++) {
        uint64_t i = it * stride + blockIdx.x * uint64_t(blockDim.x) + threadIdx.x;
        if (lane == 0) asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" :: "r"(mb), "r"(32 * 4 * 16));
        __syncwarp();
#pragma unroll
        for (int r = 0; r < 4; r++) {
            const uint64_t s = mix(i * 4 + r) % slots;
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 16, [%2];"
                         :: "r"(dst + 16 * r), "l"(buf + s * 64), "r"(mb) : "memory");
        }
        uint32_t done = 0;
        while (!done) {
            asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                         : "=r"(done) : "r"(mb), "r"(phase));
        }
        phase ^= 1;
        acc += *(uint64_t*)(sm + threadIdx.x * 64) + *(uint64_t*)(sm + threadIdx.x * 64 + 48);
        __syncwarp();
    }
    if (acc == 0x1234567) out[0] = acc;
}

template <class F>
void timeit(F f, uint64_t n, const char* name) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    f(n / 8);
    cudaEventRecord(a);
    f(n);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    cudaError_t e = cudaGetLastError();
    printf("{\"variant\": \"%s\", \"ms\": %.3f, \"Gloads_s\": %.2f, \"err\": \"%s\"}\n", name, ms, n / (ms * 1e-3) / 1e9,
           cudaGetErrorString(e));
    fflush(stdout);
}

int main(int argc, char** argv) {
    size_t bytes = 8ull << 30;
    uint64_t n = 512ull * 1000000;
    uint8_t* buf;
    uint64_t* out;
    cudaMalloc(&buf, bytes);
    cudaMalloc(&out, 64);
    cudaMemset(buf, 1, bytes);
    uint64_t slots = bytes / 64;
    cudaFuncSetAttribute(ldg, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    for (int sms : {18, 37, 74, 148}) {
        char name[64];
        snprintf(name, sizeof name, "ldg_1cta_per_sm_%d_sms", sms);
        timeit([&](uint64_t m) { ldg<<<sms, 1024, 200 * 1024>>>(buf, slots, m, out); }, n, name);
    }
    timeit([&](uint64_t m) { ldg<<<148 * 2, 1024, 0>>>(buf, slots, m, out); }, n, "ldg_2cta_per_sm_148");
    timeit([&](uint64_t m) { ldg<<<148, 512, 200 * 1024>>>(buf, slots, m, out); }, n, "ldg_512thr_per_sm_148");
    timeit([&](uint64_t m) { ldg<<<148, 256, 200 * 1024>>>(buf, slots, m, out); }, n, "ldg_256thr_per_sm_148");
    timeit([&](uint64_t m) { ldgsts<<<148 * 8, 256>>>(buf, slots, m, out); }, n, "cp.async_16B");
    timeit([&](uint64_t m) { bulk<<<148 * 8, 256>>>(buf, slots, m, out); }, n, "cp.async.bulk_16B");
    return 0;
}
