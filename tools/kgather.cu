// kgather.cu — K-GATHER calibration microbenchmark: independent
// random loads from a buffer far larger than L2, one variant per load flavour /
// width, to find the empirical random-access ceiling of this B200 and the DRAM
// bytes each flavour really moves per request (read with ncu).
//
//   ./kgather [buffer_GiB=8] [loads_M=1024]
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

template <int V>
__device__ __forceinline__ uint64_t ld(const uint8_t* p) {
    uint64_t v = 0;
    uint4 a, b;
    if (V == 0) asm volatile("ld.global.u64 %0, [%1];" : "=l"(v) : "l"(p));
    if (V == 1) asm volatile("ld.global.nc.u64 %0, [%1];" : "=l"(v) : "l"(p));
    if (V == 2) asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(v) : "l"(p));
    if (V == 3) asm volatile("ld.global.cs.u64 %0, [%1];" : "=l"(v) : "l"(p));
    if (V == 4) asm volatile("ld.global.nc.L1::no_allocate.u64 %0, [%1];" : "=l"(v) : "l"(p));
    if (V == 5) asm volatile("ld.global.cv.u64 %0, [%1];" : "=l"(v) : "l"(p));
    if (V == 6) {  // 16 B
        asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(a.x), "=r"(a.y), "=r"(a.z), "=r"(a.w) : "l"(p));
        v = a.x ^ a.w;
    }
    if (V == 7) {  // 32 B (one sector)
        asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(a.x), "=r"(a.y), "=r"(a.z), "=r"(a.w) : "l"(p));
        asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(b.x), "=r"(b.y), "=r"(b.z), "=r"(b.w) : "l"(p + 16));
        v = a.x ^ b.w;
    }
    if (V == 8) {  // 64 B (two sectors, one request per 16 B)
        for (int k = 0; k < 4; k++) {
            asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(a.x), "=r"(a.y), "=r"(a.z), "=r"(a.w) : "l"(p + 16 * k));
            v ^= a.x;
        }
    }
    if (V == 9) asm volatile("ld.global.nc.L2::64B.u64 %0, [%1];" : "=l"(v) : "l"(p));
    if (V == 10) asm volatile("ld.global.cg.L2::64B.u64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}

template <int V, int ILP>
__global__ void __launch_bounds__(256) gather(const uint8_t* __restrict__ buf, uint64_t slots, uint64_t n, uint64_t* out) {
    uint64_t acc = 0;
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n / ILP; i += stride) {
        uint64_t v[ILP];
#pragma unroll
        for (int r = 0; r < ILP; r++) {
            const uint64_t s = mix(i * ILP + r) % slots;       // random 64-B-aligned slot
            v[r] = ld<V>(buf + s * 64);
        }
#pragma unroll
        for (int r = 0; r < ILP; r++) acc += v[r];
    }
    if (acc == 0x1234567) out[0] = acc;
}

// dependent chain: each thread follows a pseudo-random pointer chain (latency-bound)
template <int V>
__global__ void __launch_bounds__(256) chase(const uint8_t* __restrict__ buf, uint64_t slots, uint64_t n, uint64_t* out) {
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    uint64_t acc = 0;
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n / 4; i += stride) {
        uint64_t s = mix(i) % slots;
        for (int d = 0; d < 4; d++) {
            uint64_t v = ld<V>(buf + s * 64);
            s = mix(v + s) % slots;
            acc += v;
        }
    }
    if (acc == 0x1234567) out[0] = acc;
}

// two independent 8-B loads at distance D from a random 4-KB-aligned base
template <int D>
__global__ void __launch_bounds__(256) pair(const uint8_t* __restrict__ buf, uint64_t pages, uint64_t n, uint64_t* out) {
    uint64_t acc = 0;
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n / 4; i += stride) {
        uint64_t v[8];
#pragma unroll
        for (int r = 0; r < 4; r++) {
            const uint64_t s = mix(i * 4 + r) % pages;
            v[2 * r] = ld<4>(buf + s * 4096);
            v[2 * r + 1] = ld<4>(buf + s * 4096 + D);
        }
#pragma unroll
        for (int r = 0; r < 8; r++) acc += v[r];
    }
    if (acc == 0x1234567) out[0] = acc;
}

// random 8-B stores (V=0 plain, 1 .cs streaming, 2 atomicMax u64, 3 red.max (no return))
template <int V>
__global__ void __launch_bounds__(256) scatter(uint8_t* __restrict__ buf, uint64_t slots, uint64_t n) {
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += stride) {
        const uint64_t s = mix(i) % slots;
        uint64_t* p = (uint64_t*)(buf + s * 64);
        if (V == 0) *p = i;
        if (V == 1) __stcs((unsigned long long*)p, (unsigned long long)i);
        if (V == 2) atomicMax((unsigned long long*)p, (unsigned long long)i);
        if (V == 3) asm volatile("red.global.max.u64 [%0], %1;" :: "l"(p), "l"(i));
    }
}

template <int V>
void run_scatter(uint8_t* buf, uint64_t bytes, uint64_t n, int grid, const char* name) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    scatter<V><<<grid, 256>>>(buf, bytes / 64, n / 8);
    cudaEventRecord(a);
    scatter<V><<<grid, 256>>>(buf, bytes / 64, n);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    printf("{\"variant\": \"%s\", \"ms\": %.3f, \"Gops_s\": %.2f}\n", name, ms, n / (ms * 1e-3) / 1e9);
}

template <int D>
void run_pair(const uint8_t* buf, uint64_t bytes, uint64_t n, uint64_t* out, int grid) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    pair<D><<<grid, 256>>>(buf, bytes / 4096, n / 8, out);
    cudaEventRecord(a);
    pair<D><<<grid, 256>>>(buf, bytes / 4096, n, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    printf("{\"variant\": \"pair\", \"distance\": %d, \"ms\": %.3f, \"Gpairs_s\": %.2f, \"Gloads_s\": %.2f}\n", D, ms,
           n / (ms * 1e-3) / 1e9, 2 * n / (ms * 1e-3) / 1e9);
}

template <int V, int ILP>
float run(const uint8_t* buf, uint64_t slots, uint64_t n, uint64_t* out, int grid, const char* name, int bytes) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    gather<V, ILP><<<grid, 256>>>(buf, slots, n / 8, out);
    cudaEventRecord(a);
    gather<V, ILP><<<grid, 256>>>(buf, slots, n, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    double gl = n / (ms * 1e-3) / 1e9;
    printf("{\"variant\": \"%s\", \"ilp\": %d, \"bytes_per_load\": %d, \"ms\": %.3f, \"Gloads_s\": %.2f, \"GBs_at_32B\": %.1f, \"GBs_at_req\": %.1f}\n",
           name, ILP, bytes, ms, gl, gl * 32, gl * bytes);
    return ms;
}

template <int V>
void run_chase(const uint8_t* buf, uint64_t slots, uint64_t n, uint64_t* out, int grid, const char* name) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    chase<V><<<grid, 256>>>(buf, slots, n / 8, out);
    cudaEventRecord(a);
    chase<V><<<grid, 256>>>(buf, slots, n, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    double gl = n / (ms * 1e-3) / 1e9;
    printf("{\"variant\": \"%s\", \"chain\": 4, \"ms\": %.3f, \"Gloads_s\": %.2f, \"GBs_at_32B\": %.1f}\n", name, ms, gl, gl * 32);
}

int main(int argc, char** argv) {
    double gib = argc > 1 ? atof(argv[1]) : 8.0;
    uint64_t n = (argc > 2 ? atoll(argv[2]) : 1024) * 1000000ull;
    const char* only = argc > 3 ? argv[3] : "";
    size_t bytes = size_t(gib * (1ull << 30));
    uint8_t* buf;
    uint64_t* out;
    cudaMalloc(&buf, bytes);
    cudaMalloc(&out, 64);
    cudaMemset(buf, 1, bytes);
    uint64_t slots = bytes / 64;
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int grid = sms * 8 * 16;
    printf("{\"buffer_GiB\": %.1f, \"loads\": %llu, \"sms\": %d}\n", gib, (unsigned long long)n, sms);
    bool all = only[0] == 0;
    if (all || only[0] == 'a') {
        run<0, 4>(buf, slots, n, out, grid, "ld.global(ca).u64", 8);
        run<1, 4>(buf, slots, n, out, grid, "ld.global.nc.u64", 8);
        run<2, 4>(buf, slots, n, out, grid, "ld.global.cg.u64", 8);
        run<3, 4>(buf, slots, n, out, grid, "ld.global.cs.u64", 8);
        run<4, 4>(buf, slots, n, out, grid, "ld.global.nc.L1::no_allocate.u64", 8);
        run<5, 4>(buf, slots, n, out, grid, "ld.global.cv.u64", 8);
        run<9, 4>(buf, slots, n, out, grid, "ld.global.nc.L2::64B.u64", 8);
        run<10, 4>(buf, slots, n, out, grid, "ld.global.cg.L2::64B.u64", 8);
        run<6, 4>(buf, slots, n, out, grid, "nc.na.v4 16B", 16);
        run<7, 4>(buf, slots, n, out, grid, "nc.na 2xv4 32B", 32);
        run<8, 2>(buf, slots, n, out, grid, "nc.na 4xv4 64B", 64);
        run<4, 1>(buf, slots, n, out, grid, "ld.global.nc.L1::no_allocate.u64", 8);
        run<4, 8>(buf, slots, n, out, grid, "ld.global.nc.L1::no_allocate.u64", 8);
        run<2, 8>(buf, slots, n, out, grid, "ld.global.cg.u64", 8);
        run_chase<1>(buf, slots, n, out, grid, "chase nc");
        run_chase<2>(buf, slots, n, out, grid, "chase cg");
        run_chase<4>(buf, slots, n, out, grid, "chase nc.na");
    }
    if (all || only[0] == 'p') {
        run_pair<8>(buf, bytes, n, out, grid);
        run_pair<64>(buf, bytes, n, out, grid);
        run_pair<128>(buf, bytes, n, out, grid);
        run_pair<256>(buf, bytes, n, out, grid);
        run_pair<512>(buf, bytes, n, out, grid);
        run_pair<1024>(buf, bytes, n, out, grid);
        run_pair<2048>(buf, bytes, n, out, grid);
    }
    if (all || only[0] == 's') {
        run_scatter<0>(buf, bytes, n, grid, "store8_random");
        run_scatter<1>(buf, bytes, n, grid, "store8_random_cs");
        run_scatter<2>(buf, bytes, n, grid, "atomicMax64_random");
        run_scatter<3>(buf, bytes, n, grid, "red.max64_random");
        run_scatter<0>(buf, 64ull << 20, n, grid, "store8_random_64MiB");
        run_scatter<2>(buf, 64ull << 20, n, grid, "atomicMax64_random_64MiB");
    }
    if (all || only[0] == 'f') {   // footprint sweep: random 8-B loads within the first F bytes
        for (uint64_t f = 16ull << 20; f <= bytes && f <= (4ull << 30); f *= 2) {
            char name[64];
            snprintf(name, sizeof name, "footprint_%lluMiB", (unsigned long long)(f >> 20));
            run<4, 4>(buf, f / 64, n, out, grid, name, 8);
        }
    }
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) printf("{\"error\": \"%s\"}\n", cudaGetErrorString(e));
    return 0;
}
