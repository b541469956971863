// bucket_micro.cu — microbenchmark of the K-BUCKET streaming kernels (bucket.cuh)
// against read / copy calibration kernels and experimental variants, on 2^30
// uniform random u64 keys (8 GiB, far larger than L2).  Prints one JSON line per
// kernel: ms (median of 5) and GB/s of compulsory bytes.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include \
//        -I paper_conf_icpp_koppehelggp21_b200/csrc tools/bucket_micro.cu -o /tmp/bm
#include <cstdio>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>
#include "bucket.cuh"
using namespace cuart;

__global__ void fill(uint64_t* q, uint64_t n) {
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x) {
        uint64_t z = i * 0x9E3779B97F4A7C15ull + 12345;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        q[i] = z ^ (z >> 31);
    }
}
__global__ void __launch_bounds__(256) rd_u64(const uint64_t* __restrict__ q, uint64_t n, uint64_t* sink) {
    const uint64_t base = uint64_t(blockIdx.x) * 4096;
    uint64_t v[16], acc = 0;
#pragma unroll
    for (int r = 0; r < 16; r++) { const uint64_t i = base + r * 256 + threadIdx.x; v[r] = i < n ? __ldcs((const unsigned long long*)q + i) : 0; }
#pragma unroll
    for (int r = 0; r < 16; r++) acc ^= v[r];
    if (acc == 0x12345) sink[0] = acc;
}
__global__ void __launch_bounds__(256) rd_v4(const uint64_t* __restrict__ q, uint64_t n, uint64_t* sink) {
    const uint64_t base = uint64_t(blockIdx.x) * 4096;
    uint4 v[8]; uint32_t acc = 0;
#pragma unroll
    for (int r = 0; r < 8; r++) { const uint64_t i = base + 2 * (r * 256 + threadIdx.x); v[r] = i < n ? __ldcs((const uint4*)(q + i)) : make_uint4(0,0,0,0); }
#pragma unroll
    for (int r = 0; r < 8; r++) acc ^= v[r].x ^ v[r].y ^ v[r].z ^ v[r].w;
    if (acc == 0x12345) sink[0] = acc;
}
__global__ void __launch_bounds__(256) cp_v4(const uint64_t* __restrict__ q, uint64_t n, uint64_t* __restrict__ o) {
    const uint64_t base = uint64_t(blockIdx.x) * 4096;
    uint4 v[8];
#pragma unroll
    for (int r = 0; r < 8; r++) { const uint64_t i = base + 2 * (r * 256 + threadIdx.x); v[r] = i < n ? __ldcs((const uint4*)(q + i)) : make_uint4(0,0,0,0); }
#pragma unroll
    for (int r = 0; r < 8; r++) { const uint64_t i = base + 2 * (r * 256 + threadIdx.x); if (i < n) __stcs((uint4*)(o + i), v[r]); }
}
// hist with 16-B loads: 8 loads of 2 keys per thread
__global__ void __launch_bounds__(256) hist_v4(const uint64_t* __restrict__ q, uint64_t n, uint32_t depth, unsigned int* __restrict__ hist) {
    __shared__ unsigned int h[kBuckets];
    h[threadIdx.x] = 0;
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    uint4 v[8];
#pragma unroll
    for (int r = 0; r < 8; r++) { const uint64_t i = base + 2 * (r * 256 + threadIdx.x); v[r] = i + 1 < n ? __ldcs((const uint4*)(q + i)) : make_uint4(0,0,0,0); }
#pragma unroll
    for (int r = 0; r < 8; r++) {
        const uint64_t i = base + 2 * (r * 256 + threadIdx.x);
        if (i < n) atomicAdd(&h[bucket_of(KeyU64{uint64_t(v[r].x) | (uint64_t(v[r].y) << 32)}, depth)], 1u);
        if (i + 1 < n) atomicAdd(&h[bucket_of(KeyU64{uint64_t(v[r].z) | (uint64_t(v[r].w) << 32)}, depth)], 1u);
    }
    __syncthreads();
    hist[hidx(threadIdx.x, blockIdx.x)] = h[threadIdx.x];
}
// gather without launch-bound cap, early jpos loads (u16 per position)
__global__ void __launch_bounds__(kBucketThreads) g_early(const uint64_t* __restrict__ res,
                                                            const uint16_t* __restrict__ jpos, uint64_t n,
                                                            const unsigned int* __restrict__ rowoff,
                                                            const unsigned int* __restrict__ bases,
                                                            uint64_t* __restrict__ out) {
    __shared__ uint64_t sres[kBucketTile];
    __shared__ uint8_t bof[kBucketTile];
    __shared__ unsigned int loc[kBuckets];
    __shared__ unsigned int glb[kBuckets];
    __shared__ unsigned int wtot[kBucketThreads / 32];
    const uint64_t t = blockIdx.x, tiles = gridDim.x;
    const uint64_t base = t * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    const int b = threadIdx.x;
    const unsigned int off = rowoff[hidx(b, t)];
    const unsigned int bb = bases[b];
    const unsigned int bnext = b + 1 < kBuckets ? bases[b + 1] : unsigned(n);
    const unsigned int next = t + 1 < tiles ? rowoff[hidx(b, t + 1)] : bnext - bb;
    uint16_t jp[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) { const uint32_t k = uint32_t(r) * kBucketThreads + threadIdx.x; jp[r] = k < cnt ? __ldcs(jpos + base + k) : 0; }
    const unsigned int c_b = next - off;
    glb[b] = bb + off;
    const unsigned int l_b = block_excl_scan256(c_b, wtot);
    loc[b] = l_b;
    for (unsigned int k = 0; k < c_b; k++) bof[l_b + k] = uint8_t(b);
    __syncthreads();
    uint64_t v[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * kBucketThreads + threadIdx.x;
        v[r] = 0;
        if (j < cnt) { const uint32_t bj = bof[j]; v[r] = __ldcs((const unsigned long long*)res + glb[bj] + (j - loc[bj])); }
    }
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) { const uint32_t j = uint32_t(r) * kBucketThreads + threadIdx.x; if (j < cnt) sres[j] = v[r]; }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) { const uint32_t k = uint32_t(r) * kBucketThreads + threadIdx.x; if (k < cnt) __stcs((unsigned long long*)out + base + k, (unsigned long long)sres[jp[r]]); }
}
__global__ void __launch_bounds__(kBucketThreads) g_old(const uint64_t* __restrict__ res,
                                                            const uint16_t* __restrict__ jpos, uint64_t n,
                                                            const unsigned int* __restrict__ rowoff,
                                                            const unsigned int* __restrict__ bases,
                                                            uint64_t* __restrict__ out) {
    __shared__ uint64_t sres[kBucketTile];
    __shared__ uint8_t bof[kBucketTile];                               // bucket of each tile-local position
    __shared__ unsigned int loc[kBuckets];
    __shared__ unsigned int glb[kBuckets];
    __shared__ unsigned int wtot[kBucketThreads / 32];
    const uint64_t t = blockIdx.x, tiles = gridDim.x;
    const uint64_t base = t * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    const int b = threadIdx.x;
    const unsigned int off = rowoff[hidx(b, t)];
    const unsigned int btotal = (b + 1 < kBuckets ? bases[b + 1] : unsigned(n)) - bases[b];
    const unsigned int next = t + 1 < tiles ? rowoff[hidx(b, t + 1)] : btotal;
    const unsigned int c_b = next - off;
    glb[b] = bases[b] + off;
    const unsigned int l_b = block_excl_scan256(c_b, wtot);
    loc[b] = l_b;
    for (unsigned int k = 0; k < c_b; k++) bof[l_b + k] = uint8_t(b);
    __syncthreads();
    uint64_t v[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {                           // 16 independent loads in flight
        const uint32_t j = uint32_t(r) * kBucketThreads + threadIdx.x;
        v[r] = 0;
        if (j < cnt) {
            const uint32_t bj = bof[j];
            v[r] = __ldcs((const unsigned long long*)res + glb[bj] + (j - loc[bj]));
        }
    }
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * kBucketThreads + threadIdx.x;
        if (j < cnt) sres[j] = v[r];
    }
    __syncthreads();
    uint32_t jp[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t k = uint32_t(r) * kBucketThreads + threadIdx.x;
        jp[r] = k < cnt ? __ldcs(jpos + base + k) : 0u;
    }
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t k = uint32_t(r) * kBucketThreads + threadIdx.x;
        if (k < cnt) __stcs((unsigned long long*)out + base + k, (unsigned long long)sres[jp[r]]);
    }
}



__device__ __forceinline__ void cp_async16(void* smem, const void* g) {
    const unsigned sa = unsigned(__cvta_generic_to_shared(smem));
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(sa), "l"(g));
}
__device__ __forceinline__ void cp_async_wait() {
    asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
}
// gather: runs copied into smem with cp.async (no registers held), early jpos loads
__global__ void __launch_bounds__(kBucketThreads) g_ca(const uint64_t* __restrict__ res,
                                                            const uint16_t* __restrict__ jpos, uint64_t n,
                                                            const unsigned int* __restrict__ rowoff,
                                                            const unsigned int* __restrict__ bases,
                                                            uint64_t* __restrict__ out) {
    __shared__ uint64_t sres[kBucketTile];
    __shared__ uint8_t bof[kBucketTile];
    __shared__ unsigned int loc[kBuckets];
    __shared__ unsigned int glb[kBuckets];
    __shared__ unsigned int wtot[kBucketThreads / 32];
    const uint64_t t = blockIdx.x, tiles = gridDim.x;
    const uint64_t base = t * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    const int b = threadIdx.x;
    const unsigned int off = rowoff[hidx(b, t)];
    const unsigned int bb = bases[b];
    const unsigned int bnext = b + 1 < kBuckets ? bases[b + 1] : unsigned(n);
    const unsigned int next = t + 1 < tiles ? rowoff[hidx(b, t + 1)] : bnext - bb;
    uint16_t jp[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) { const uint32_t k = uint32_t(r) * kBucketThreads + threadIdx.x; jp[r] = k < cnt ? __ldcs(jpos + base + k) : 0; }
    const unsigned int c_b = next - off;
    glb[b] = bb + off;
    const unsigned int l_b = block_excl_scan256(c_b, wtot);
    loc[b] = l_b;
    for (unsigned int k = 0; k < c_b; k++) bof[l_b + k] = uint8_t(b);
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * kBucketThreads + threadIdx.x;
        if (j < cnt) { const uint32_t bj = bof[j]; cp_async8(&sres[j], res + glb[bj] + (j - loc[bj])); }
    }
    cp_async_wait();
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) { const uint32_t k = uint32_t(r) * kBucketThreads + threadIdx.x; if (k < cnt) __stcs((unsigned long long*)out + base + k, (unsigned long long)sres[jp[r]]); }
}
// scatter: keys copied into smem in original order with cp.async (16 B = 2 keys per
// copy); buckets from smem; staged position -> original position table; copy phase
// reads skeys[sidx[j]].
__global__ void __launch_bounds__(kBucketThreads) s_ca(const uint64_t* __restrict__ q, uint64_t n, uint32_t depth,
                                                       const unsigned int* __restrict__ rowoff,
                                                       const unsigned int* __restrict__ bases,
                                                       uint64_t* __restrict__ bq, uint16_t* __restrict__ jpos) {
    __shared__ __align__(16) uint64_t skeys[kBucketTile];
    __shared__ uint16_t sidx[kBucketTile];
    __shared__ uint8_t sb[kBucketTile];
    __shared__ unsigned int h[kBuckets];
    __shared__ unsigned int loc[kBuckets];
    __shared__ unsigned int glb[kBuckets];
    __shared__ unsigned int wtot[kBucketThreads / 32];
    h[threadIdx.x] = 0;
    const unsigned int gb = bases[threadIdx.x] + rowoff[hidx(threadIdx.x, blockIdx.x)];
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
#pragma unroll
    for (int r = 0; r < kBucketItems / 2; r++) {
        const uint32_t j = 2 * (uint32_t(r) * kBucketThreads + threadIdx.x);
        if (j + 1 < cnt) cp_async16(&skeys[j], q + base + j);
        else if (j < cnt) cp_async8(&skeys[j], q + base + j);
    }
    cp_async_wait();
    __syncthreads();
    uint32_t br[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * kBucketThreads + threadIdx.x;
        br[r] = 0xFFFFFFFFu;
        if (j < cnt) { const uint32_t bk = bucket_of(KeyU64{skeys[j]}, depth); br[r] = (bk << 16) | atomicAdd(&h[bk], 1u); }
    }
    __syncthreads();
    loc[threadIdx.x] = block_excl_scan256(h[threadIdx.x], wtot);
    glb[threadIdx.x] = gb;
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t jt = uint32_t(r) * kBucketThreads + threadIdx.x;
        if (br[r] != 0xFFFFFFFFu) {
            const uint32_t bk = br[r] >> 16, j = loc[bk] + (br[r] & 0xFFFFu);
            sb[j] = uint8_t(bk);
            sidx[j] = uint16_t(jt);
            __stcs((unsigned short*)jpos + base + jt, (unsigned short)j);
        }
    }
    __syncthreads();
#pragma unroll 4
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * kBucketThreads + threadIdx.x;
        if (j < cnt) { const uint32_t bk = sb[j]; __stcs((unsigned long long*)bq + glb[bk] + (j - loc[bk]), (unsigned long long)skeys[sidx[j]]); }
    }
}
// scatter with 16-B key loads (keys in registers, as the product kernel otherwise)
__global__ void __launch_bounds__(kBucketThreads) s_v4(const uint64_t* __restrict__ q, uint64_t n, uint32_t depth,
                                                       const unsigned int* __restrict__ rowoff,
                                                       const unsigned int* __restrict__ bases,
                                                       uint64_t* __restrict__ bq, uint16_t* __restrict__ jpos) {
    __shared__ __align__(16) uint64_t skeys[kBucketTile];
    __shared__ uint8_t sb[kBucketTile];
    __shared__ unsigned int h[kBuckets];
    __shared__ unsigned int loc[kBuckets];
    __shared__ unsigned int glb[kBuckets];
    __shared__ unsigned int wtot[kBucketThreads / 32];
    h[threadIdx.x] = 0;
    const unsigned int gb = bases[threadIdx.x] + rowoff[hidx(threadIdx.x, blockIdx.x)];
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    uint4 v[kBucketItems / 2];
#pragma unroll
    for (int r = 0; r < kBucketItems / 2; r++) {
        const uint32_t j = 2 * (uint32_t(r) * kBucketThreads + threadIdx.x);
        v[r] = j + 1 < cnt ? __ldcs((const uint4*)(q + base + j)) : make_uint4(0, 0, 0, 0);
        if (j + 1 == cnt) { const uint64_t x = __ldcs((const unsigned long long*)q + base + j); v[r].x = uint32_t(x); v[r].y = uint32_t(x >> 32); }
    }
    __syncthreads();
    uint32_t br[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = 2 * ((uint32_t(r) >> 1) * kBucketThreads + threadIdx.x) + (r & 1);
        br[r] = 0xFFFFFFFFu;
        const uint4 w = v[r >> 1];
        const uint64_t key = (r & 1) ? (uint64_t(w.z) | (uint64_t(w.w) << 32)) : (uint64_t(w.x) | (uint64_t(w.y) << 32));
        if (j < cnt) { const uint32_t bk = bucket_of(KeyU64{key}, depth); br[r] = (bk << 16) | atomicAdd(&h[bk], 1u); }
    }
    __syncthreads();
    loc[threadIdx.x] = block_excl_scan256(h[threadIdx.x], wtot);
    glb[threadIdx.x] = gb;
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t jt = 2 * ((uint32_t(r) >> 1) * kBucketThreads + threadIdx.x) + (r & 1);
        if (br[r] != 0xFFFFFFFFu) {
            const uint32_t bk = br[r] >> 16, j = loc[bk] + (br[r] & 0xFFFFu);
            const uint4 w = v[r >> 1];
            skeys[j] = (r & 1) ? (uint64_t(w.z) | (uint64_t(w.w) << 32)) : (uint64_t(w.x) | (uint64_t(w.y) << 32));
            sb[j] = uint8_t(bk);
            __stcs((unsigned short*)jpos + base + jt, (unsigned short)j);
        }
    }
    __syncthreads();
#pragma unroll 4
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * kBucketThreads + threadIdx.x;
        if (j < cnt) { const uint32_t bk = sb[j]; __stcs((unsigned long long*)bq + glb[bk] + (j - loc[bk]), (unsigned long long)skeys[j]); }
    }
}

// scatter / gather with more threads per 4096-key tile (THREADS x 4096/THREADS items):
// more warps per SM to overlap the CTA phases (load -> rank -> scan -> stage -> copy)
__device__ __forceinline__ unsigned int scan256_wide(unsigned int v, unsigned int* wtot) {
    // exclusive scan over threads 0..255 (callers pass v for those); all threads sync
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    unsigned int x = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const unsigned int y = __shfl_up_sync(0xffffffffu, x, d);
        if (lane >= d) x += y;
    }
    if (lane == 31 && warp < 8) wtot[warp] = x;
    __syncthreads();
    unsigned int before = 0;
#pragma unroll
    for (int w = 0; w < 8; w++) before += w < warp ? wtot[w] : 0u;
    return before + x - v;
}
template <int THREADS>
__global__ void __launch_bounds__(THREADS) s_wide(const uint64_t* __restrict__ q, uint64_t n, uint32_t depth,
                                                  const unsigned int* __restrict__ rowoff, const unsigned int* __restrict__ bases,
                                                  uint64_t* __restrict__ bq, uint16_t* __restrict__ jpos) {
    constexpr int ITEMS = kBucketTile / THREADS;
    __shared__ uint64_t skeys[kBucketTile];
    __shared__ uint8_t sb[kBucketTile];
    __shared__ unsigned int h[kBuckets], loc[kBuckets], glb[kBuckets], wtot[8];
    const int t = threadIdx.x;
    unsigned int gb = 0;
    if (t < kBuckets) { h[t] = 0; gb = bases[t] + rowoff[hidx(t, blockIdx.x)]; }
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    uint64_t kv[ITEMS];
    uint32_t br[ITEMS];
#pragma unroll
    for (int r = 0; r < ITEMS; r++) {
        const uint32_t j = uint32_t(r) * THREADS + t;
        kv[r] = j < cnt ? uint64_t(__ldcs((const unsigned long long*)q + base + j)) : 0;
    }
#pragma unroll
    for (int r = 0; r < ITEMS; r++) {
        const uint32_t j = uint32_t(r) * THREADS + t;
        br[r] = 0xFFFFFFFFu;
        if (j < cnt) { const uint32_t b = bucket_of(KeyU64{kv[r]}, depth); br[r] = (b << 16) | atomicAdd(&h[b], 1u); }
    }
    __syncthreads();
    const unsigned int mine = t < kBuckets ? h[t] : 0u;
    const unsigned int lb = scan256_wide(mine, wtot);
    if (t < kBuckets) { loc[t] = lb; glb[t] = gb - lb; }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < ITEMS; r++) {
        const uint32_t jt = uint32_t(r) * THREADS + t;
        if (br[r] != 0xFFFFFFFFu) {
            const uint32_t b = br[r] >> 16, j = loc[b] + (br[r] & 0xFFFFu);
            sb[j] = uint8_t(b);
            skeys[j] = kv[r];
            __stcs((unsigned short*)jpos + base + jt, (unsigned short)j);
        }
    }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < ITEMS; r++) {
        const uint32_t j = uint32_t(r) * THREADS + t;
        if (j < cnt) __stcs((unsigned long long*)bq + uint64_t(glb[sb[j]] + j), (unsigned long long)skeys[j]);
    }
}
template <int THREADS>
__global__ void __launch_bounds__(THREADS) g_wide(const uint64_t* __restrict__ res, const uint16_t* __restrict__ jpos, uint64_t n,
                                                  const unsigned int* __restrict__ rowoff, const unsigned int* __restrict__ bases,
                                                  uint64_t* __restrict__ out) {
    constexpr int ITEMS = kBucketTile / THREADS;
    __shared__ uint64_t sres[kBucketTile];
    __shared__ uint8_t bof[kBucketTile];
    __shared__ unsigned int loc[kBuckets], glb[kBuckets], wtot[8];
    const uint64_t tb = blockIdx.x, tiles = gridDim.x;
    const uint64_t base = tb * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    const int t = threadIdx.x;
    uint16_t jp[ITEMS];
#pragma unroll
    for (int r = 0; r < ITEMS; r++) {
        const uint32_t k = uint32_t(r) * THREADS + t;
        jp[r] = k < cnt ? __ldcs(jpos + base + k) : 0;
    }
    unsigned int c_b = 0, off = 0, bb = 0;
    if (t < kBuckets) {
        off = rowoff[hidx(t, tb)];
        bb = bases[t];
        const unsigned int bnext = t + 1 < kBuckets ? bases[t + 1] : unsigned(n);
        const unsigned int next = tb + 1 < tiles ? rowoff[hidx(t, tb + 1)] : bnext - bb;
        c_b = next - off;
    }
    const unsigned int l_b = scan256_wide(c_b, wtot);
    if (t < kBuckets) {
        glb[t] = bb + off;
        loc[t] = l_b;
        for (unsigned int k = 0; k < c_b; k++) bof[l_b + k] = uint8_t(t);
    }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < ITEMS; r++) {
        const uint32_t j = uint32_t(r) * THREADS + t;
        if (j < cnt) { const uint32_t bj = bof[j]; cp_async8(&sres[j], res + glb[bj] + (j - loc[bj])); }
    }
    cp_async_wait_all();
    __syncthreads();
#pragma unroll
    for (int r = 0; r < ITEMS; r++) {
        const uint32_t k = uint32_t(r) * THREADS + t;
        if (k < cnt) __stcs((unsigned long long*)out + base + k, (unsigned long long)sres[jp[r]]);
    }
}

// ---- persistent scatter with TMA bulk tile loads (double-buffered, mbarrier-signalled)
__device__ __forceinline__ uint32_t saddr(const void* p) { return uint32_t(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(saddr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, uint64_t* bar) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(saddr(bar)), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(saddr(dst)), "l"(src), "r"(bytes), "r"(saddr(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, unsigned parity) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}"
                     : "=r"(ok) : "r"(saddr(bar)), "r"(parity) : "memory");
}
constexpr size_t kTmaScatterSmem = 2 * kBucketTile * 8 + kBucketTile * 8 + kBucketTile + 64;
__global__ void __launch_bounds__(256) s_tma(const uint64_t* __restrict__ q, uint64_t n, uint32_t depth,
                                             const unsigned int* __restrict__ rowoff, const unsigned int* __restrict__ bases,
                                             uint64_t* __restrict__ bq, uint16_t* __restrict__ jpos) {
    extern __shared__ __align__(128) uint8_t sm[];
    uint64_t* kin = (uint64_t*)sm;                                   // [2][kBucketTile]
    uint64_t* skeys = kin + 2 * kBucketTile;                         // staged tile
    uint8_t* sb = (uint8_t*)(skeys + kBucketTile);
    uint64_t* bar = (uint64_t*)(sb + kBucketTile);                   // [2]
    __shared__ unsigned int h[kBuckets], loc[kBuckets], glb[kBuckets], wtot[8];
    const int t = threadIdx.x;
    const uint64_t tiles = (n + kBucketTile - 1) / kBucketTile;
    const uint64_t full_tiles = n / kBucketTile;                     // tiles loaded by TMA
    if (t == 0) {
        mbar_init(&bar[0], 1);
        mbar_init(&bar[1], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    uint64_t tile = blockIdx.x;
    if (t == 0 && tile < full_tiles) bulk_g2s(kin, q + tile * kBucketTile, kBucketTile * 8, &bar[0]);
    for (uint32_t it = 0; tile < tiles; it++, tile += gridDim.x) {
        const uint32_t buf = it & 1;
        const uint64_t nxt = tile + gridDim.x;
        if (t == 0 && nxt < full_tiles) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            bulk_g2s(kin + (buf ^ 1) * kBucketTile, q + nxt * kBucketTile, kBucketTile * 8, &bar[buf ^ 1]);
        }
        const unsigned int gb = bases[t] + rowoff[hidx(t, tile)];
        h[t] = 0;
        const uint64_t base = tile * kBucketTile;
        const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
        const uint64_t* kt = kin + buf * kBucketTile;
        if (tile < full_tiles) mbar_wait(&bar[buf], (it >> 1) & 1);
        else for (uint32_t j = t; j < cnt; j += 256) ((uint64_t*)kt)[j] = q[base + j];
        __syncthreads();
        uint32_t br[kBucketItems];
#pragma unroll
        for (int r = 0; r < kBucketItems; r++) {
            const uint32_t j = uint32_t(r) * 256 + t;
            br[r] = 0xFFFFFFFFu;
            if (j < cnt) { const uint32_t b = bucket_of(KeyU64{kt[j]}, depth); br[r] = (b << 16) | atomicAdd(&h[b], 1u); }
        }
        __syncthreads();
        const unsigned int lb = block_excl_scan256(h[t], wtot);
        loc[t] = lb;
        glb[t] = gb - lb;
        __syncthreads();
#pragma unroll
        for (int r = 0; r < kBucketItems; r++) {
            const uint32_t jt = uint32_t(r) * 256 + t;
            if (br[r] != 0xFFFFFFFFu) {
                const uint32_t b = br[r] >> 16, j = loc[b] + (br[r] & 0xFFFFu);
                sb[j] = uint8_t(b);
                skeys[j] = kt[jt];
                __stcs((unsigned short*)jpos + base + jt, (unsigned short)j);
            }
        }
        __syncthreads();
#pragma unroll 4
        for (int r = 0; r < kBucketItems; r++) {
            const uint32_t j = uint32_t(r) * 256 + t;
            if (j < cnt) __stcs((unsigned long long*)bq + uint64_t(glb[sb[j]] + j), (unsigned long long)skeys[j]);
        }
        __syncthreads();
    }
}

// scatter without the per-position bucket byte: the copy phase recomputes the bucket
// from the staged key (one shift) instead of a random smem byte store + a byte load
__global__ void __launch_bounds__(256, 4) s_nosb(const uint64_t* __restrict__ q, uint64_t n, uint32_t depth,
                                              const unsigned int* __restrict__ rowoff, const unsigned int* __restrict__ bases,
                                              uint64_t* __restrict__ bq, uint16_t* __restrict__ jpos) {
    __shared__ uint64_t skeys[kBucketTile];
    __shared__ unsigned int h[kBuckets], loc[kBuckets], glb[kBuckets], wtot[8];
    const int t = threadIdx.x;
    h[t] = 0;
    const unsigned int gb = bases[t] + rowoff[hidx(t, blockIdx.x)];
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    uint64_t kv[kBucketItems];
    uint32_t br[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * 256 + t;
        kv[r] = j < cnt ? uint64_t(__ldcs((const unsigned long long*)q + base + j)) : 0;
    }
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * 256 + t;
        br[r] = 0xFFFFFFFFu;
        if (j < cnt) { const uint32_t b = bucket_of(KeyU64{kv[r]}, depth); br[r] = (b << 16) | atomicAdd(&h[b], 1u); }
    }
    __syncthreads();
    const unsigned int lb = block_excl_scan256(h[t], wtot);
    loc[t] = lb;
    glb[t] = gb - lb;
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t jt = uint32_t(r) * 256 + t;
        if (br[r] != 0xFFFFFFFFu) {
            const uint32_t b = br[r] >> 16, j = loc[b] + (br[r] & 0xFFFFu);
            skeys[j] = kv[r];
            __stcs((unsigned short*)jpos + base + jt, (unsigned short)j);
        }
    }
    __syncthreads();
#pragma unroll 4
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * 256 + t;
        if (j < cnt) {
            const uint64_t kk = skeys[j];
            __stcs((unsigned long long*)bq + uint64_t(glb[bucket_of(KeyU64{kk}, depth)] + j), (unsigned long long)kk);
        }
    }
}

__global__ void __launch_bounds__(256, 4) s_match(const uint64_t* __restrict__ q, uint64_t n, uint32_t depth,
                                              const unsigned int* __restrict__ rowoff, const unsigned int* __restrict__ bases,
                                              uint64_t* __restrict__ bq, uint16_t* __restrict__ jpos) {
    __shared__ uint64_t skeys[kBucketTile];
    __shared__ unsigned int h[kBuckets], loc[kBuckets], glb[kBuckets], wtot[8];
    const int t = threadIdx.x;
    h[t] = 0;
    const unsigned int gb = bases[t] + rowoff[hidx(t, blockIdx.x)];
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    uint64_t kv[kBucketItems];
    uint32_t br[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * 256 + t;
        kv[r] = j < cnt ? uint64_t(__ldcs((const unsigned long long*)q + base + j)) : 0;
    }
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * 256 + t;
        br[r] = 0xFFFFFFFFu;
        const uint32_t b = j < cnt ? bucket_of(KeyU64{kv[r]}, depth) : 0xFFFFu;   // inactive lanes: own group
        const unsigned peers = __match_any_sync(0xffffffffu, b);
        const unsigned lane = threadIdx.x & 31u;
        const int leader = __ffs(peers) - 1;
        unsigned basev = 0;
        if (int(lane) == leader && b != 0xFFFFu) basev = atomicAdd(&h[b], unsigned(__popc(peers)));
        basev = __shfl_sync(0xffffffffu, basev, leader);
        if (j < cnt) br[r] = (b << 16) | (basev + __popc(peers & ((1u << lane) - 1u)));
    }
    __syncthreads();
    const unsigned int lb = block_excl_scan256(h[t], wtot);
    loc[t] = lb;
    glb[t] = gb - lb;
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t jt = uint32_t(r) * 256 + t;
        if (br[r] != 0xFFFFFFFFu) {
            const uint32_t b = br[r] >> 16, j = loc[b] + (br[r] & 0xFFFFu);
            skeys[j] = kv[r];
            __stcs((unsigned short*)jpos + base + jt, (unsigned short)j);
        }
    }
    __syncthreads();
#pragma unroll 4
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * 256 + t;
        if (j < cnt) {
            const uint64_t kk = skeys[j];
            __stcs((unsigned long long*)bq + uint64_t(glb[bucket_of(KeyU64{kk}, depth)] + j), (unsigned long long)kk);
        }
    }
}

__global__ void __launch_bounds__(256, 4) s_seqw(const uint64_t* __restrict__ q, uint64_t n, uint32_t depth,
                                              const unsigned int* __restrict__ rowoff, const unsigned int* __restrict__ bases,
                                              uint64_t* __restrict__ bq, uint16_t* __restrict__ jpos) {
    __shared__ uint64_t skeys[kBucketTile];
    __shared__ unsigned int h[kBuckets], loc[kBuckets], glb[kBuckets], wtot[8];
    const int t = threadIdx.x;
    h[t] = 0;
    const unsigned int gb = bases[t] + rowoff[hidx(t, blockIdx.x)];
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    uint64_t kv[kBucketItems];
    uint32_t br[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * 256 + t;
        kv[r] = j < cnt ? uint64_t(__ldcs((const unsigned long long*)q + base + j)) : 0;
    }
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * 256 + t;
        br[r] = 0xFFFFFFFFu;
        if (j < cnt) { const uint32_t b = bucket_of(KeyU64{kv[r]}, depth); br[r] = (b << 16) | atomicAdd(&h[b], 1u); }
    }
    __syncthreads();
    const unsigned int lb = block_excl_scan256(h[t], wtot);
    loc[t] = lb;
    glb[t] = gb - lb;
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t jt = uint32_t(r) * 256 + t;
        if (br[r] != 0xFFFFFFFFu) {
            const uint32_t b = br[r] >> 16, j = loc[b] + (br[r] & 0xFFFFu);
            skeys[j] = kv[r];
            __stcs((unsigned short*)jpos + base + jt, (unsigned short)j);
        }
    }
    __syncthreads();
#pragma unroll 4
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * 256 + t;
        if (j < cnt) {
            const uint64_t kk = skeys[j];
            __stcs((unsigned long long*)bq + base + j, (unsigned long long)(kk + glb[bucket_of(KeyU64{kk}, depth)]));
        }
    }
}

// diagnostic: one global atomicAdd per (tile, bucket) on 256 counters spread STRIDE words apart
template <int STRIDE>
__global__ void __launch_bounds__(256) atom_alloc(unsigned int* fill, unsigned int* sink) {
    const unsigned int v = atomicAdd(&fill[threadIdx.x * STRIDE], 16u + (blockIdx.x & 3));
    if (v == 0xFFFFFFFFu) sink[0] = v;
}

// ---- tile of 8192 keys (512 threads x 16): runs twice as long (avg 32 keys = 256 B per
// bucket run), half the hist entries
constexpr int kBigThreads = 512, kBigTile = kBigThreads * kBucketItems;
__global__ void __launch_bounds__(kBigThreads) h_big(const uint64_t* __restrict__ q, uint64_t n, uint32_t depth, unsigned int* __restrict__ hist) {
    __shared__ unsigned int h[kBuckets];
    const int t = threadIdx.x;
    if (t < kBuckets) h[t] = 0;
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kBigTile;
    uint4 v[kBucketItems / 2];
#pragma unroll
    for (int r = 0; r < kBucketItems / 2; r++) {
        const uint64_t i = base + 2 * (uint64_t(r) * kBigThreads + t);
        v[r] = i + 2 <= n ? __ldcs((const uint4*)(q + i)) : make_uint4(0, 0, 0, 0);
    }
#pragma unroll
    for (int r = 0; r < kBucketItems / 2; r++) {
        const uint64_t i = base + 2 * (uint64_t(r) * kBigThreads + t);
        if (i + 2 <= n) {
            atomicAdd(&h[bucket_of(KeyU64{uint64_t(v[r].x) | (uint64_t(v[r].y) << 32)}, depth)], 1u);
            atomicAdd(&h[bucket_of(KeyU64{uint64_t(v[r].z) | (uint64_t(v[r].w) << 32)}, depth)], 1u);
        } else if (i < n) atomicAdd(&h[bucket_of(KeyU64{q[i]}, depth)], 1u);
    }
    __syncthreads();
    if (t < kBuckets) hist[hidx(t, blockIdx.x)] = h[t];
}
__global__ void __launch_bounds__(kBigThreads) s_big(const uint64_t* __restrict__ q, uint64_t n, uint32_t depth,
                                                     const unsigned int* __restrict__ rowoff, const unsigned int* __restrict__ bases,
                                                     uint64_t* __restrict__ bq, uint16_t* __restrict__ jpos) {
    extern __shared__ __align__(16) uint64_t skeys[];
    __shared__ unsigned int h[kBuckets], loc[kBuckets], glb[kBuckets], wtot[8];
    const int t = threadIdx.x;
    unsigned int gb = 0;
    if (t < kBuckets) { h[t] = 0; gb = bases[t] + rowoff[hidx(t, blockIdx.x)]; }
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kBigTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBigTile) ? n - base : kBigTile);
    uint64_t kv[kBucketItems];
    uint32_t br[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * kBigThreads + t;
        kv[r] = j < cnt ? uint64_t(__ldcs((const unsigned long long*)q + base + j)) : 0;
    }
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * kBigThreads + t;
        br[r] = 0xFFFFFFFFu;
        if (j < cnt) { const uint32_t b = bucket_of(KeyU64{kv[r]}, depth); br[r] = (b << 16) | atomicAdd(&h[b], 1u); }
    }
    __syncthreads();
    const unsigned int lb = scan256_wide(t < kBuckets ? h[t] : 0u, wtot);
    if (t < kBuckets) { loc[t] = lb; glb[t] = gb - lb; }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t jt = uint32_t(r) * kBigThreads + t;
        if (br[r] != 0xFFFFFFFFu) {
            const uint32_t b = br[r] >> 16, j = loc[b] + (br[r] & 0xFFFFu);
            skeys[j] = kv[r];
            __stcs((unsigned short*)jpos + base + jt, (unsigned short)j);
        }
    }
    __syncthreads();
#pragma unroll 4
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * kBigThreads + t;
        if (j < cnt) {
            const uint64_t kk = skeys[j];
            __stcs((unsigned long long*)bq + uint64_t(glb[bucket_of(KeyU64{kk}, depth)] + j), (unsigned long long)kk);
        }
    }
}
__global__ void __launch_bounds__(kBigThreads) g_big(const uint64_t* __restrict__ res, const uint16_t* __restrict__ jpos, uint64_t n,
                                                     const unsigned int* __restrict__ rowoff, const unsigned int* __restrict__ bases,
                                                     uint64_t* __restrict__ out) {
    extern __shared__ __align__(16) uint64_t sres[];
    uint8_t* bof = (uint8_t*)(sres + kBigTile);
    __shared__ unsigned int loc[kBuckets], glb[kBuckets], wtot[8];
    const uint64_t tb = blockIdx.x, tiles = gridDim.x;
    const uint64_t base = tb * kBigTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBigTile) ? n - base : kBigTile);
    const int t = threadIdx.x;
    uint16_t jp[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t k = uint32_t(r) * kBigThreads + t;
        jp[r] = k < cnt ? __ldcs(jpos + base + k) : 0;
    }
    unsigned int c_b = 0, off = 0, bb = 0;
    if (t < kBuckets) {
        off = rowoff[hidx(t, tb)];
        bb = bases[t];
        const unsigned int bnext = t + 1 < kBuckets ? bases[t + 1] : unsigned(n);
        const unsigned int next = tb + 1 < tiles ? rowoff[hidx(t, tb + 1)] : bnext - bb;
        c_b = next - off;
    }
    const unsigned int l_b = scan256_wide(c_b, wtot);
    if (t < kBuckets) {
        glb[t] = bb + off;
        loc[t] = l_b;
        for (unsigned int k = 0; k < c_b; k++) bof[l_b + k] = uint8_t(t);
    }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * kBigThreads + t;
        if (j < cnt) { const uint32_t bj = bof[j]; cp_async8(&sres[j], res + glb[bj] + (j - loc[bj])); }
    }
    cp_async_wait_all();
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t k = uint32_t(r) * kBigThreads + t;
        if (k < cnt) __stcs((unsigned long long*)out + base + k, (unsigned long long)sres[jp[r]]);
    }
}

__global__ void csum(const uint64_t* a, uint64_t n, unsigned long long* s) {
    uint64_t acc = 0;
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x) acc += a[i] * (i | 1);
    atomicAdd(s, (unsigned long long)acc);
}

template <class F>
static void timeit(const char* name, double bytes, F f) {
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    std::vector<float> ms;
    for (int rep = 0; rep < 6; rep++) {
        cudaEventRecord(e0); f(); cudaEventRecord(e1); cudaEventSynchronize(e1);
        float m; cudaEventElapsedTime(&m, e0, e1); if (rep) ms.push_back(m);
    }
    std::sort(ms.begin(), ms.end());
    const double m = ms[ms.size() / 2];
    printf("{\"kernel\": \"%s\", \"ms\": %.4f, \"GBps\": %.1f, \"err\": \"%s\"}\n", name, m, bytes / m / 1e6, cudaGetErrorString(cudaGetLastError()));
    fflush(stdout);
}
static unsigned long long checksum(const uint64_t* a, uint64_t n) {
    unsigned long long* s; cudaMalloc(&s, 8); cudaMemset(s, 0, 8);
    csum<<<1184, 256>>>(a, n, s);
    unsigned long long h; cudaMemcpy(&h, s, 8, cudaMemcpyDeviceToHost); cudaFree(s); return h;
}

int main(int argc, char** argv) {
    const uint64_t n = (argc > 1) ? strtoull(argv[1], 0, 0) : (uint64_t(1) << 30);
    const uint64_t tiles = (n + kBucketTile - 1) / kBucketTile;
    uint64_t *q, *bq, *res, *out, *sink; uint16_t* jpos; unsigned int *hist, *tot;
    cudaMalloc(&q, n * 8); cudaMalloc(&bq, n * 8); cudaMalloc(&res, n * 8); cudaMalloc(&out, n * 8);
    cudaMalloc(&jpos, n * 2); cudaMalloc(&hist, hist_entries(tiles) * 4); cudaMalloc(&tot, 1024); cudaMalloc(&sink, 8);
    fill<<<1184, 256>>>(q, n);
    fill<<<1184, 256>>>(res, n);
    const size_t smem = bscatter_smem<KeyU64>();
    cudaFuncSetAttribute(k_bscatter<KeyU64>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    const unsigned T = unsigned(tiles);
    timeit("rd_u64", n * 8.0, [&] { rd_u64<<<T, 256>>>(q, n, sink); });
    timeit("rd_v4", n * 8.0, [&] { rd_v4<<<T, 256>>>(q, n, sink); });
    timeit("cp_v4", n * 16.0, [&] { cp_v4<<<T, 256>>>(q, n, out); });
    timeit("hist_v4", n * 8.0, [&] { hist_v4<<<T, 256>>>(q, n, 0, hist); });
    timeit("k_bhist", n * 8.0, [&] { k_bhist<KeyU64, true><<<T, 256>>>(q, nullptr, n, 0, hist); });
    timeit("k_bscan_rows", hist_entries(tiles) * 8.0, [&] { k_bhist<KeyU64, true><<<T, 256>>>(q, nullptr, n, 0, hist); k_bscan_rows<<<kBuckets, kBucketThreads>>>(hist, tiles, tot); });
    k_bhist<KeyU64, true><<<T, 256>>>(q, nullptr, n, 0, hist);
    k_bscan_rows<<<kBuckets, kBucketThreads>>>(hist, tiles, tot);
    k_bscan<<<1, kBuckets>>>(tot, kBuckets);
    timeit("k_bscatter", n * 18.0, [&] { k_bscatter<KeyU64><<<T, 256, smem>>>(q, nullptr, n, 0, hist, tot, bq, nullptr, jpos); });
    timeit("k_bgather", n * 18.0, [&] { k_bgather<false><<<T, 256>>>(res, jpos, n, hist, tot, out); });
    const unsigned long long c1 = checksum(out, n);
    timeit("g_old", n * 18.0, [&] { g_old<<<T, 256>>>(res, jpos, n, hist, tot, out); });
    const unsigned long long c2 = checksum(out, n);
    timeit("g_early", n * 18.0, [&] { g_early<<<T, 256>>>(res, jpos, n, hist, tot, out); });
    const unsigned long long c3 = checksum(out, n);
    timeit("g_ca", n * 18.0, [&] { g_ca<<<T, 256>>>(res, jpos, n, hist, tot, out); });
    const unsigned long long c4 = checksum(out, n);
    printf("{\"gather_checksums_equal\": %s}\n", (c1 == c2 && c2 == c3 && c3 == c4) ? "true" : "false");
    // scatter variants: each must reproduce the bucketed batch as a multiset per bucket;
    // compare checksums of bq (order inside a tile's run may differ: atomics rank)
    const unsigned long long s0 = checksum(bq, n);
    timeit("s_ca", n * 18.0, [&] { s_ca<<<T, 256>>>(q, n, 0, hist, tot, bq, jpos); });
    timeit("g_ca_after_s_ca", n * 18.0, [&] { g_ca<<<T, 256>>>(bq, jpos, n, hist, tot, out); });
    const unsigned long long s1 = checksum(out, n), s1b = checksum(q, n);
    timeit("s_v4", n * 18.0, [&] { s_v4<<<T, 256>>>(q, n, 0, hist, tot, bq, jpos); });
    g_ca<<<T, 256>>>(bq, jpos, n, hist, tot, out);
    const unsigned long long s2 = checksum(out, n);
    timeit("k_bscatter_again", n * 18.0, [&] { k_bscatter<KeyU64><<<T, 256, smem>>>(q, nullptr, n, 0, hist, tot, bq, nullptr, jpos); });
    k_bgather<false><<<T, 256>>>(bq, jpos, n, hist, tot, out);
    const unsigned long long s3 = checksum(out, n);
    for (int v = 0; v < 2; v++) {
        const char* sn = v == 0 ? "s_wide512" : "s_wide1024";
        const char* gn = v == 0 ? "g_wide512" : "g_wide1024";
        timeit(sn, n * 18.0, [&] { if (v == 0) s_wide<512><<<T, 512>>>(q, n, 0, hist, tot, bq, jpos); else s_wide<1024><<<T, 1024>>>(q, n, 0, hist, tot, bq, jpos); });
        timeit(gn, n * 18.0, [&] { if (v == 0) g_wide<512><<<T, 512>>>(bq, jpos, n, hist, tot, out); else g_wide<1024><<<T, 1024>>>(bq, jpos, n, hist, tot, out); });
        printf("{\"roundtrip_%s\": %s}\n", sn, checksum(out, n) == s1b ? "true" : "false");
    }
    timeit("s_nosb", n * 18.0, [&] { s_nosb<<<T, 256>>>(q, n, 0, hist, tot, bq, jpos); });
    g_ca<<<T, 256>>>(bq, jpos, n, hist, tot, out);
    printf("{\"roundtrip_s_nosb\": %s}\n", checksum(out, n) == s1b ? "true" : "false");
    timeit("s_match (match_any ranking, 256 buckets)", n * 18.0, [&] { s_match<<<T, 256>>>(q, n, 0, hist, tot, bq, jpos); });
    g_ca<<<T, 256>>>(bq, jpos, n, hist, tot, out);
    printf("{\"roundtrip_s_match\": %s}\n", checksum(out, n) == s1b ? "true" : "false");
    {   // 64 buckets (root byte >> 2), as the product default for c3
        const uint32_t d64 = 2u << 8;
        k_bhist<KeyU64, true><<<T, 256>>>(q, nullptr, n, d64, hist);
        k_bscan_rows<<<kBuckets, kBucketThreads>>>(hist, tiles, tot);
        k_bscan<<<1, kBuckets>>>(tot, kBuckets);
        timeit("k_bscatter_64", n * 18.0, [&] { k_bscatter<KeyU64><<<T, 256, smem>>>(q, nullptr, n, d64, hist, tot, bq, nullptr, jpos); });
        timeit("k_bgather_64", n * 18.0, [&] { k_bgather<false><<<T, 256>>>(bq, jpos, n, hist, tot, out); });
        printf("{\"roundtrip_64\": %s}\n", checksum(out, n) == s1b ? "true" : "false");
        timeit("s_match_64", n * 18.0, [&] { s_match<<<T, 256>>>(q, n, d64, hist, tot, bq, jpos); });
        k_bgather<false><<<T, 256>>>(bq, jpos, n, hist, tot, out);
        printf("{\"roundtrip_s_match_64\": %s}\n", checksum(out, n) == s1b ? "true" : "false");
        k_bhist<KeyU64, true><<<T, 256>>>(q, nullptr, n, 0, hist);
        k_bscan_rows<<<kBuckets, kBucketThreads>>>(hist, tiles, tot);
        k_bscan<<<1, kBuckets>>>(tot, kBuckets);
    }
    {
        unsigned int* fill; cudaMalloc(&fill, 256 * 1024 * 4); cudaMemset(fill, 0, 256 * 1024 * 4);
        timeit("atom_alloc_stride1", 0, [&] { atom_alloc<1><<<T, 256>>>(fill, (unsigned int*)sink); });
        timeit("atom_alloc_stride64", 0, [&] { atom_alloc<64><<<T, 256>>>(fill, (unsigned int*)sink); });
        timeit("atom_alloc_stride1024", 0, [&] { atom_alloc<1024><<<T, 256>>>(fill, (unsigned int*)sink); });
        cudaFree(fill);
    }
    timeit("s_seqw (diagnostic: sequential writes)", n * 18.0, [&] { s_seqw<<<T, 256>>>(q, n, 0, hist, tot, bq, jpos); });
    cudaFuncSetAttribute(s_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, int(kTmaScatterSmem));
    for (int cps = 1; cps <= 2; cps++) {
        char nm[32];
        snprintf(nm, sizeof nm, "s_tma_x%d", cps);
        int nsm = 0;
        cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
        timeit(nm, n * 18.0, [&] { s_tma<<<nsm * cps, 256, kTmaScatterSmem>>>(q, n, 0, hist, tot, bq, jpos); });
        g_ca<<<T, 256>>>(bq, jpos, n, hist, tot, out);
        printf("{\"roundtrip_%s\": %s}\n", nm, checksum(out, n) == s1b ? "true" : "false");
    }
    {
        const uint64_t tb = (n + kBigTile - 1) / kBigTile;
        const size_t ss = size_t(kBigTile) * 8, gs = size_t(kBigTile) * 9;
        cudaFuncSetAttribute(s_big, cudaFuncAttributeMaxDynamicSharedMemorySize, int(ss));
        cudaFuncSetAttribute(g_big, cudaFuncAttributeMaxDynamicSharedMemorySize, int(gs));
        timeit("h_big", n * 8.0, [&] { h_big<<<unsigned(tb), kBigThreads>>>(q, n, 0, hist); });
        k_bscan_rows<<<kBuckets, kBucketThreads>>>(hist, tb, tot);
        k_bscan<<<1, kBuckets>>>(tot, kBuckets);
        timeit("s_big", n * 18.0, [&] { s_big<<<unsigned(tb), kBigThreads, ss>>>(q, n, 0, hist, tot, bq, jpos); });
        timeit("g_big", n * 18.0, [&] { g_big<<<unsigned(tb), kBigThreads, gs>>>(bq, jpos, n, hist, tot, out); });
        printf("{\"roundtrip_big\": %s}\n", checksum(out, n) == s1b ? "true" : "false");
    }
    printf("{\"roundtrip_s_v4\": %s, \"roundtrip_k_bscatter\": %s}\n", s2 == s1b ? "true" : "false", s3 == s1b ? "true" : "false");
    printf("{\"s0\": %llu, \"roundtrip_ok\": %s}\n", s0, s1 == s1b ? "true" : "false");
    return 0;
}
