// route.cu — K-ROUTE / K-UNROUTE for the range-partitioned multi-GPU layer
// (SURVEY §8(e)).  The key space is split by P-1 splitters over the first 8 key
// bytes (big-endian, so numeric order = lexicographic order, reading C2); the
// owner of a key is the number of splitters <= its 8-byte prefix.  A batch is
// scattered into per-owner contiguous runs, STABLE in op order, so that an
// owner receiving the runs of all sources concatenated by source rank sees the
// ops in global (rank-major) order — the order the update semantics need
// (the highest op index wins; reading C7).
//
//   k_route_hist   : owner of every op (kept in scratch) + per-block histogram
//   k_route_scan   : exclusive offsets per (owner, block) + per-owner counts
//   k_route_scatter: stable per-owner placement via warp ballots; perm[i] = slot
//   k_unroute      : out[i] = results[perm[i]]
//
// The multi-GPU layer proper (cuart_dist_*, csrc/dist.cu) fuses routing into the
// K-BUCKET pass; these standalone kernels remain the general partition primitive
// (cuart_partition_by_flag splits config 5's mixed rounds, reading C7).
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <cstring>

#include "../../include/cuart.h"
#include "layout.h"

namespace {

constexpr int kRouteThreads = 256;
constexpr int kRouteItems = 16;                 // ops per thread per block
constexpr int kRouteChunk = kRouteThreads * kRouteItems;
constexpr uint32_t kMaxParts = 64;

__device__ __forceinline__ uint64_t load_prefix8(uint32_t kind, const void* keys, const uint8_t* lens, uint64_t i) {
    if (kind == CUART_KEY_U64) return ((const uint64_t*)keys)[i];
    if (kind == CUART_KEY_U32) return uint64_t(((const uint32_t*)keys)[i]) << 32;
    const uint8_t* s = (const uint8_t*)keys + i * 32;
    const uint32_t l = lens[i];
    uint64_t p = 0;
#pragma unroll
    for (int b = 0; b < 8; b++) p = (p << 8) | (uint32_t(b) < l ? s[b] : 0u);
    return p;
}

__device__ __forceinline__ uint32_t owner_of(uint64_t prefix, const uint64_t* sp, uint32_t nsp) {
    uint32_t lo = 0, hi = nsp;                  // number of splitters <= prefix
    while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (sp[mid] <= prefix) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

__global__ void __launch_bounds__(kRouteThreads) k_route_hist(uint32_t kind, const void* __restrict__ keys,
                                                              const uint8_t* __restrict__ lens, uint64_t n,
                                                              const uint64_t* __restrict__ splitters, uint32_t nparts,
                                                              const uint8_t* __restrict__ flags,
                                                              uint8_t* __restrict__ owner, uint32_t* __restrict__ hist) {
    __shared__ uint64_t sp[kMaxParts];
    __shared__ uint32_t h[kMaxParts];
    for (uint32_t t = threadIdx.x; t < kMaxParts; t += blockDim.x) {
        if (splitters && t + 1 < nparts) sp[t] = splitters[t];
        h[t] = 0;
    }
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kRouteChunk;
    for (int r = 0; r < kRouteItems; r++) {
        const uint64_t i = base + uint64_t(r) * kRouteThreads + threadIdx.x;
        if (i < n) {
            const uint32_t o = flags ? (flags[i] ? 1u : 0u) : owner_of(load_prefix8(kind, keys, lens, i), sp, nparts - 1);
            owner[i] = uint8_t(o);
            atomicAdd(&h[o], 1u);
        }
    }
    __syncthreads();
    for (uint32_t o = threadIdx.x; o < nparts; o += blockDim.x) hist[uint64_t(o) * gridDim.x + blockIdx.x] = h[o];
}

// Single CTA: exclusive scan of hist in (owner, block) order -> offsets, counts.
__global__ void __launch_bounds__(1024) k_route_scan(uint32_t* __restrict__ hist, uint64_t nblocks, uint32_t nparts,
                                                     uint64_t* __restrict__ counts) {
    __shared__ uint64_t warp_sums[32];
    __shared__ uint64_t carry;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    const uint64_t total = nblocks * nparts;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (uint64_t start = 0; start < total; start += blockDim.x) {
        const uint64_t idx = start + threadIdx.x;
        const uint64_t v = idx < total ? hist[idx] : 0;
        uint64_t x = v;                                   // inclusive warp scan
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint64_t y = __shfl_up_sync(0xffffffffu, x, d);
            if (lane >= d) x += y;
        }
        if (lane == 31) warp_sums[warp] = x;
        __syncthreads();
        if (warp == 0) {
            uint64_t w = lane < int(blockDim.x >> 5) ? warp_sums[lane] : 0;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint64_t y = __shfl_up_sync(0xffffffffu, w, d);
                if (lane >= d) w += y;
            }
            warp_sums[lane] = w;
        }
        __syncthreads();
        const uint64_t excl = carry + (warp ? warp_sums[warp - 1] : 0) + x - v;
        if (idx < total) hist[idx] = uint32_t(excl);      // offsets fit 32 bits (n < 2^32 per call)
        __syncthreads();
        if (threadIdx.x == blockDim.x - 1) carry = excl + v;
        __syncthreads();
    }
    // counts[o] = offset of owner o+1 - offset of owner o
    for (uint32_t o = threadIdx.x; o < nparts; o += blockDim.x) {
        const uint64_t beg = hist[uint64_t(o) * nblocks];
        const uint64_t end = (o + 1 < nparts) ? hist[uint64_t(o + 1) * nblocks] : carry;
        counts[o] = end - beg;
    }
}

__global__ void __launch_bounds__(kRouteThreads) k_route_scatter(uint32_t kind, const void* __restrict__ keys,
                                                                 const uint8_t* __restrict__ lens,
                                                                 const uint64_t* __restrict__ values, uint64_t n,
                                                                 uint32_t nparts, const uint8_t* __restrict__ owner,
                                                                 const uint32_t* __restrict__ offsets,
                                                                 void* __restrict__ send_keys, uint8_t* __restrict__ send_lens,
                                                                 uint64_t* __restrict__ send_values,
                                                                 uint32_t* __restrict__ perm) {
    constexpr int kWarps = kRouteThreads / 32;
    __shared__ uint32_t run[kMaxParts];             // placed so far in this block, per owner
    __shared__ uint32_t wcnt[kWarps][kMaxParts];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (uint32_t o = threadIdx.x; o < nparts; o += blockDim.x) {
        run[o] = offsets[uint64_t(o) * gridDim.x + blockIdx.x];
    }
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kRouteChunk;
    const uint32_t lt = (1u << lane) - 1;
    for (int r = 0; r < kRouteItems; r++) {
        const uint64_t i = base + uint64_t(r) * kRouteThreads + threadIdx.x;
        const bool valid = i < n;
        const uint32_t o = valid ? owner[i] : 0xFFFFFFFFu;
        // per-owner ballots: warp counts, and this lane's rank among same-owner lanes
        uint32_t rank = 0;
        for (uint32_t oo = 0; oo < nparts; oo++) {
            const uint32_t m = __ballot_sync(0xffffffffu, o == oo);
            if (o == oo) rank = __popc(m & lt);
            if (lane == 0) wcnt[warp][oo] = __popc(m);
        }
        __syncthreads();
        if (valid) {
            uint32_t before = 0;
            for (int w = 0; w < warp; w++) before += wcnt[w][o];
            const uint32_t slot = run[o] + before + rank;
            perm[i] = slot;
            const uint64_t dst = uint64_t(slot);
            void* kd = send_keys;
            if (kind == CUART_KEY_U64) ((uint64_t*)kd)[dst] = ((const uint64_t*)keys)[i];
            else if (kind == CUART_KEY_U32) ((uint32_t*)kd)[dst] = ((const uint32_t*)keys)[i];
            else {
                const uint4* s = (const uint4*)keys + 2 * i;
                uint4* d = (uint4*)kd + 2 * dst;
                d[0] = s[0];
                d[1] = s[1];
                send_lens[dst] = lens[i];
            }
            if (values) send_values[dst] = values[i];
        }
        __syncthreads();
        for (uint32_t oo = threadIdx.x; oo < nparts; oo += blockDim.x) {
            uint32_t tot = 0;
            for (int w = 0; w < kWarps; w++) tot += wcnt[w][oo];
            run[oo] += tot;
        }
        __syncthreads();
    }
}

__global__ void __launch_bounds__(256) k_unroute(const uint64_t* __restrict__ in, const uint32_t* __restrict__ perm,
                                                 uint64_t n, uint64_t* __restrict__ out) {
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += stride) out[i] = in[perm[i]];
}

// ---- two-way stable partition by flag (cuart_partition_by_flag) ------------
// Ops with flag 0 first, then flag != 0, each in op order.  A thread owns 16
// CONSECUTIVE ops of a 4096-op tile, so one block scan of the per-thread counts
// ranks the whole tile (no per-round barriers): k_pf_count counts the tile's flag-0
// ops (16-B flag loads), k_pf_scan turns the counts into tile offsets, k_pf_scatter
// places every op at (flag 0) off0[tile] + rank or (flag 1) L + (tile base - off0[tile])
// + rank.  Streaming bytes per u64 op: 1 (count) + 1 + 8 + 8 read, 8 + 8 + 4 written.
constexpr int kPfPer = kRouteChunk / kRouteThreads;     // 16 consecutive ops per thread

__device__ __forceinline__ uint32_t zero_flag_count16(uint4 v) {
    uint32_t c = 0;
#pragma unroll
    for (int w = 0; w < 4; w++) {
        const uint32_t x = (&v.x)[w];
#pragma unroll
        for (int b = 0; b < 4; b++) c += ((x >> (8 * b)) & 0xFFu) == 0 ? 1u : 0u;
    }
    return c;
}

// block-wide exclusive scan of one value per thread (256 threads); total -> *tot
__device__ __forceinline__ uint32_t pf_block_scan(uint32_t v, uint32_t* wsum, uint32_t* tot) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint32_t x = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, d);
        if (lane >= d) x += y;
    }
    if (lane == 31) wsum[warp] = x;
    __syncthreads();
    uint32_t before = 0, all = 0;
#pragma unroll
    for (int w = 0; w < kRouteThreads / 32; w++) {
        before += w < warp ? wsum[w] : 0u;
        all += wsum[w];
    }
    if (tot) *tot = all;
    return before + x - v;
}

__device__ __forceinline__ uint4 pf_flags16(const uint8_t* flags, uint64_t i, uint64_t n) {
    if (i + kPfPer <= n && (uintptr_t(flags + i) & 15) == 0) return *(const uint4*)(flags + i);
    uint4 v = make_uint4(0x01010101u, 0x01010101u, 0x01010101u, 0x01010101u);   // past the end: "flag 1", never placed
    for (int e = 0; e < kPfPer; e++)
        if (i + e < n) {
            const uint32_t sh = 8 * (e & 3);
            uint32_t& w = (&v.x)[e >> 2];
            w = (w & ~(0xFFu << sh)) | (uint32_t(flags[i + e]) << sh);
        }
    return v;
}

__global__ void __launch_bounds__(kRouteThreads) k_pf_count(const uint8_t* __restrict__ flags, uint64_t n,
                                                            uint32_t* __restrict__ cnt0) {
    __shared__ uint32_t wsum[kRouteThreads / 32];
    __shared__ uint32_t tot;
    const uint64_t i = uint64_t(blockIdx.x) * kRouteChunk + uint64_t(threadIdx.x) * kPfPer;
    const uint32_t c = i < n ? zero_flag_count16(pf_flags16(flags, i, n)) : 0u;
    pf_block_scan(c, wsum, threadIdx.x == 0 ? &tot : nullptr);
    if (threadIdx.x == 0) cnt0[blockIdx.x] = tot;
}

// One CTA: exclusive scan of the per-tile flag-0 counts (in place) + counts[0..1].
__global__ void __launch_bounds__(1024) k_pf_scan(uint32_t* __restrict__ cnt0, uint64_t ntiles, uint64_t n,
                                                  uint64_t* __restrict__ counts) {
    __shared__ uint64_t wsum[32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t per = (ntiles + 1023) / 1024;
    const uint64_t t0 = uint64_t(threadIdx.x) * per;
    uint64_t s = 0;
    for (uint64_t t = t0; t < t0 + per && t < ntiles; t++) s += cnt0[t];
    uint64_t x = s;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint64_t y = __shfl_up_sync(0xffffffffu, x, d);
        if (lane >= d) x += y;
    }
    if (lane == 31) wsum[warp] = x;
    __syncthreads();
    uint64_t before = 0, all = 0;
    for (int w = 0; w < 32; w++) {
        before += w < warp ? wsum[w] : 0;
        all += wsum[w];
    }
    uint64_t run = before + x - s;
    for (uint64_t t = t0; t < t0 + per && t < ntiles; t++) {
        const uint32_t c = cnt0[t];
        cnt0[t] = uint32_t(run);
        run += c;
    }
    if (threadIdx.x == 0) {
        counts[0] = all;
        counts[1] = n - all;
    }
}

__global__ void __launch_bounds__(kRouteThreads) k_pf_scatter(uint32_t kind, const void* __restrict__ keys,
                                                              const uint8_t* __restrict__ lens,
                                                              const uint64_t* __restrict__ values, uint64_t n,
                                                              const uint8_t* __restrict__ flags,
                                                              const uint32_t* __restrict__ off0,
                                                              const uint64_t* __restrict__ counts,
                                                              void* __restrict__ out_keys, uint8_t* __restrict__ out_lens,
                                                              uint64_t* __restrict__ out_values,
                                                              uint32_t* __restrict__ perm) {
    __shared__ uint32_t wsum[kRouteThreads / 32];
    __shared__ uint32_t sdst[kRouteChunk];                            // destination slot of every op of the tile
    const uint64_t tb = uint64_t(blockIdx.x) * kRouteChunk;
    const uint64_t i0 = tb + uint64_t(threadIdx.x) * kPfPer;
    const uint4 fv = pf_flags16(flags, i0, n);
    const uint32_t c0 = i0 < n ? zero_flag_count16(fv) : 0u;
    const uint32_t r0 = pf_block_scan(c0, wsum, nullptr);             // flag-0 ops before mine in the tile
    const uint64_t L = counts[0];
    const uint64_t b0 = off0[blockIdx.x];                              // flag-0 ops before this tile
    // slots relative to the partition's flag-0 / flag-1 bases fit 32 bits (n < 2^32)
    uint32_t p0 = uint32_t(b0 + r0);                                   // next flag-0 slot
    uint32_t p1 = uint32_t(L + (tb - b0) + (uint64_t(threadIdx.x) * kPfPer - r0));   // next flag-1 slot
#pragma unroll
    for (int e = 0; e < kPfPer; e++) {
        const bool f = (((&fv.x)[e >> 2] >> (8 * (e & 3))) & 0xFFu) != 0;
        sdst[threadIdx.x * kPfPer + e] = f ? p1++ : p0++;
    }
    __syncthreads();
    // the copy: op j of the tile in coalesced order; runs of equal flags land in
    // consecutive slots, so the stores are coalesced too
#pragma unroll 4
    for (int r = 0; r < kPfPer; r++) {
        const uint32_t j = uint32_t(r) * kRouteThreads + threadIdx.x;
        const uint64_t i = tb + j;
        if (i >= n) break;
        const uint64_t dst = sdst[j];
        perm[i] = uint32_t(dst);
        if (kind == CUART_KEY_U64) ((uint64_t*)out_keys)[dst] = ((const uint64_t*)keys)[i];
        else if (kind == CUART_KEY_U32) ((uint32_t*)out_keys)[dst] = ((const uint32_t*)keys)[i];
        else {
            const uint4* src = (const uint4*)keys + 2 * i;
            uint4* d = (uint4*)out_keys + 2 * dst;
            d[0] = src[0];
            d[1] = src[1];
            out_lens[dst] = lens[i];
        }
        if (values) out_values[dst] = values[i];
    }
}

// out[i] = in[perm[i]], 4 ops per thread (16-B perm loads and 32-B stores when aligned)
__global__ void __launch_bounds__(256) k_unroute4(const uint64_t* __restrict__ in, const uint32_t* __restrict__ perm,
                                                  uint64_t n, uint64_t* __restrict__ out) {
    const uint64_t i = (uint64_t(blockIdx.x) * 256 + threadIdx.x) * 4;
    if (i + 4 <= n) {
        const uint4 p = __ldcs((const uint4*)(perm + i));
        const uint64_t a = in[p.x], b = in[p.y], c = in[p.z], d = in[p.w];
        __stcs((ulonglong2*)(out + i), make_ulonglong2(a, b));
        __stcs((ulonglong2*)(out + i) + 1, make_ulonglong2(c, d));
    } else {
        for (uint64_t j = i; j < n; j++) out[j] = in[perm[j]];
    }
}

}  // namespace

extern std::atomic<uint64_t> g_cuart_launches;

extern "C" {

size_t cuart_route_scratch_bytes(size_t n, uint32_t nparts) {
    const uint64_t nblocks = (n + kRouteChunk - 1) / kRouteChunk;
    return ((n + 255) & ~size_t(255)) + nblocks * nparts * sizeof(uint32_t) + 256;
}

static cuart_status route_impl(const cuart_keys* keys, size_t n, const uint64_t* splitters, const uint8_t* flags,
                               uint32_t nparts, const uint64_t* values, void* send_keys, uint8_t* send_lengths,
                               uint64_t* send_values, uint32_t* perm, uint64_t* counts, void* scratch, void* stream);

cuart_status cuart_route(const cuart_keys* keys, size_t n, const uint64_t* splitters, uint32_t nparts,
                         const uint64_t* values, void* send_keys, uint8_t* send_lengths, uint64_t* send_values,
                         uint32_t* perm, uint64_t* counts, void* scratch, void* stream) {
    if (nparts > 1 && !splitters) return CUART_ERR_INVALID_ARGUMENT;
    return route_impl(keys, n, splitters, nullptr, nparts, values, send_keys, send_lengths, send_values, perm, counts,
                      scratch, stream);
}

cuart_status cuart_partition_by_flag(const cuart_keys* keys, size_t n, const uint8_t* flags, const uint64_t* values,
                                     void* out_keys, uint8_t* out_lengths, uint64_t* out_values, uint32_t* perm,
                                     uint64_t* counts, void* scratch, void* stream) {
    if (n > 0 && !flags) return CUART_ERR_INVALID_ARGUMENT;
    if (!keys || !counts) return CUART_ERR_INVALID_ARGUMENT;
    if (n >= (uint64_t(1) << 32)) return CUART_ERR_INVALID_ARGUMENT;
    cudaStream_t s = (cudaStream_t)stream;
    if (n == 0) return cudaMemsetAsync(counts, 0, 2 * sizeof(uint64_t), s) == cudaSuccess ? CUART_OK : CUART_ERR_CUDA;
    if (!keys->data || !out_keys || !perm || !scratch) return CUART_ERR_INVALID_ARGUMENT;
    if (keys->kind == CUART_KEY_BYTES && (!keys->lengths || !out_lengths)) return CUART_ERR_INVALID_ARGUMENT;
    if (values && !out_values) return CUART_ERR_INVALID_ARGUMENT;
    const uint64_t ntiles = (n + kRouteChunk - 1) / kRouteChunk;
    uint32_t* cnt0 = (uint32_t*)((uint8_t*)scratch + ((n + 255) & ~size_t(255)));   // the route histogram's space
    const uint32_t kind = uint32_t(keys->kind);
    k_pf_count<<<unsigned(ntiles), kRouteThreads, 0, s>>>(flags, n, cnt0);
    k_pf_scan<<<1, 1024, 0, s>>>(cnt0, ntiles, n, counts);
    k_pf_scatter<<<unsigned(ntiles), kRouteThreads, 0, s>>>(kind, keys->data, keys->lengths, values, n, flags, cnt0,
                                                            counts, out_keys, out_lengths, out_values, perm);
    g_cuart_launches += 3;
    return cudaGetLastError() == cudaSuccess ? CUART_OK : CUART_ERR_CUDA;
}

static cuart_status route_impl(const cuart_keys* keys, size_t n, const uint64_t* splitters, const uint8_t* flags,
                               uint32_t nparts, const uint64_t* values, void* send_keys, uint8_t* send_lengths,
                               uint64_t* send_values, uint32_t* perm, uint64_t* counts, void* scratch, void* stream) {
    if (!keys || nparts == 0 || nparts > kMaxParts || !counts) return CUART_ERR_INVALID_ARGUMENT;
    if (n >= (uint64_t(1) << 32)) return CUART_ERR_INVALID_ARGUMENT;
    cudaStream_t s = (cudaStream_t)stream;
    if (n == 0) {
        if (cudaMemsetAsync(counts, 0, nparts * sizeof(uint64_t), s) != cudaSuccess) return CUART_ERR_CUDA;
        return CUART_OK;
    }
    if (!keys->data || !send_keys || !perm || !scratch) return CUART_ERR_INVALID_ARGUMENT;
    if (keys->kind == CUART_KEY_BYTES && (!keys->lengths || !send_lengths)) return CUART_ERR_INVALID_ARGUMENT;
    if (values && !send_values) return CUART_ERR_INVALID_ARGUMENT;
    const uint64_t nblocks = (n + kRouteChunk - 1) / kRouteChunk;
    uint8_t* owner = (uint8_t*)scratch;
    uint32_t* hist = (uint32_t*)((uint8_t*)scratch + ((n + 255) & ~size_t(255)));
    const uint32_t kind = uint32_t(keys->kind);
    k_route_hist<<<unsigned(nblocks), kRouteThreads, 0, s>>>(kind, keys->data, keys->lengths, n, splitters, nparts,
                                                             flags, owner, hist);
    k_route_scan<<<1, 1024, 0, s>>>(hist, nblocks, nparts, counts);
    k_route_scatter<<<unsigned(nblocks), kRouteThreads, 0, s>>>(kind, keys->data, keys->lengths, values, n,
                                                                       nparts, owner, hist, send_keys, send_lengths,
                                                                       send_values, perm);
    g_cuart_launches += 3;
    return cudaGetLastError() == cudaSuccess ? CUART_OK : CUART_ERR_CUDA;
}

cuart_status cuart_fill_miss(uint64_t* out, size_t n, void* stream) {
    if (n == 0) return CUART_OK;
    if (!out) return CUART_ERR_INVALID_ARGUMENT;
    return cudaMemsetAsync(out, 0xFF, n * 8, (cudaStream_t)stream) == cudaSuccess ? CUART_OK : CUART_ERR_CUDA;
}

cuart_status cuart_unroute(const uint64_t* in, const uint32_t* perm, size_t n, uint64_t* out, void* stream) {
    if (n == 0) return CUART_OK;
    if (!in || !perm || !out) return CUART_ERR_INVALID_ARGUMENT;
    if ((uintptr_t(perm) & 15) == 0 && (uintptr_t(out) & 15) == 0 && (n + 1023) / 1024 < (uint64_t(1) << 31)) {
        k_unroute4<<<unsigned((n + 1023) / 1024), 256, 0, (cudaStream_t)stream>>>(in, perm, n, out);
        g_cuart_launches += 1;
        return cudaGetLastError() == cudaSuccess ? CUART_OK : CUART_ERR_CUDA;
    }
    uint64_t blocks = (n + 255) / 256;
    if (blocks > (uint64_t(1) << 31) - 1) blocks = (uint64_t(1) << 31) - 1;
    k_unroute<<<unsigned(blocks), 256, 0, (cudaStream_t)stream>>>(in, perm, n, out);
    g_cuart_launches += 1;
    return cudaGetLastError() == cudaSuccess ? CUART_OK : CUART_ERR_CUDA;
}

}  // extern "C"

// ============================================================================ range queries
// §8(f) f2 (§3.2.1): leaves are strictly lexicographic inside each leaf
// buffer, so the answer to a range query [lo, hi] is the pair of leaf indices
// (start, end) = (#leaves with key < lo, #leaves with key <= hi).  Integer keys
// live in the leaf8 buffer only; both bounds come from a branch-free binary search
// over that buffer (the top levels of the implicit search tree stay L2-resident).
// Deleted leaves keep their key bytes and position (tombstone value).
namespace {

__device__ __forceinline__ uint64_t bswap64_r(uint64_t x) {
    uint32_t lo = uint32_t(x), hi = uint32_t(x >> 32);
    return (uint64_t(__byte_perm(lo, 0, 0x0123)) << 32) | __byte_perm(hi, 0, 0x0123);
}

// number of leaf8 keys (numeric, fixed length flen) < q (strict) or <= q
__device__ __forceinline__ uint64_t rank8(const uint8_t* leaves, uint64_t nleaves, uint32_t flen, uint64_t q, bool le) {
    uint64_t lo = 0, hi = nleaves;
    while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        uint64_t k = bswap64_r(__ldg((const unsigned long long*)(leaves + mid * cuart::record_bytes(cuart::T_LEAF8))));
        if (flen == 4) k >>= 32;
        if (k < q || (le && k == q)) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

__global__ void __launch_bounds__(256) k_range(const uint8_t* __restrict__ leaves, uint64_t nleaves, uint32_t kind,
                                               const void* __restrict__ lo, const void* __restrict__ hi, uint64_t n,
                                               uint64_t* __restrict__ bounds) {
    const uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint32_t flen = kind == CUART_KEY_U64 ? 8 : 4;
    const uint64_t ql = kind == CUART_KEY_U64 ? ((const uint64_t*)lo)[i] : ((const uint32_t*)lo)[i];
    const uint64_t qh = kind == CUART_KEY_U64 ? ((const uint64_t*)hi)[i] : ((const uint32_t*)hi)[i];
    const uint64_t s = rank8(leaves, nleaves, flen, ql, false);
    uint64_t e = rank8(leaves, nleaves, flen, qh, true);
    if (e < s) e = s;                               // empty range when hi < lo
    uint64_t* b = bounds + 6 * i;
    b[0] = s;
    b[1] = e;
    b[2] = b[3] = b[4] = b[5] = 0;                  // leaf16 / leaf32 buffers are unused by integer keys
}

}  // namespace

extern "C" cuart_status cuart_range_leaf8(const uint8_t* leaves, uint64_t nleaves, uint32_t kind, const void* lo,
                                          const void* hi, size_t n, uint64_t* bounds, void* stream) {
    if (n == 0) return CUART_OK;
    const uint64_t blocks = (n + 255) / 256;
    k_range<<<unsigned(blocks), 256, 0, (cudaStream_t)stream>>>(leaves, nleaves, kind, lo, hi, n, bounds);
    g_cuart_launches += 1;
    return cudaGetLastError() == cudaSuccess ? CUART_OK : CUART_ERR_CUDA;
}

// Byte-string keys (every leaf class buffer is in lexicographic order).  The
// zero-padded bytes decide the order of two keys unless they agree on all 32 bytes;
// then the shorter key (a proper prefix) comes first -- for that the library keeps
// the key length of every leaf (leaf_len, uploaded with BYTES indexes).
namespace {

struct RangeLeaves {
    const uint8_t* rec[3];       // leaf8 / leaf16 / leaf32 records
    const uint8_t* len[3];       // their key lengths
    uint64_t count[3];
};

__device__ __forceinline__ int cmp_leaf(const uint8_t* rec, uint32_t width, uint32_t lk, const uint8_t* q, uint32_t lq) {
    for (uint32_t b = 0; b < 32; b++) {
        const uint32_t kb = b < width ? rec[b] : 0u;
        const uint32_t qb = b < lq ? q[b] : 0u;            // query bytes past its length are ignored
        if (kb != qb) return kb < qb ? -1 : 1;
    }
    return lk < lq ? -1 : (lk > lq ? 1 : 0);
}

// number of leaves of one class with key < q (le = false) or <= q (le = true)
__device__ uint64_t rank_bytes(const RangeLeaves& L, int c, const uint8_t* q, uint32_t lq, bool le) {
    const uint32_t width = c == 0 ? 8u : c == 1 ? 16u : 32u;
    const uint64_t rb = cuart::record_bytes(uint32_t(cuart::T_LEAF8 + c));
    uint64_t lo = 0, hi = L.count[c];
    while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        const int r = cmp_leaf(L.rec[c] + mid * rb, width, L.len[c][mid], q, lq);
        if (r < 0 || (le && r == 0)) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

__global__ void __launch_bounds__(128) k_range_bytes(RangeLeaves L, const uint8_t* __restrict__ lo,
                                                     const uint8_t* __restrict__ llo, const uint8_t* __restrict__ hi,
                                                     const uint8_t* __restrict__ lhi, uint64_t n,
                                                     uint64_t* __restrict__ bounds) {
    const uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (i >= n) return;
    uint8_t ql[32], qh[32];
#pragma unroll
    for (int b = 0; b < 32; b++) {
        ql[b] = lo[32 * i + b];
        qh[b] = hi[32 * i + b];
    }
    const uint32_t a = llo[i] < 32 ? llo[i] : 32u, z = lhi[i] < 32 ? lhi[i] : 32u;
    uint64_t* out = bounds + 6 * i;
    for (int c = 0; c < 3; c++) {
        const uint64_t s = rank_bytes(L, c, ql, a, false);
        uint64_t e = rank_bytes(L, c, qh, z, true);
        out[2 * c] = s;
        out[2 * c + 1] = e < s ? s : e;                    // empty range when hi < lo
    }
}

}  // namespace

extern "C" cuart_status cuart_range_bytes(const uint8_t* const* rec, const uint8_t* const* len, const uint64_t* count,
                                          const uint8_t* lo, const uint8_t* llo, const uint8_t* hi,
                                          const uint8_t* lhi, size_t n, uint64_t* bounds, void* stream) {
    if (n == 0) return CUART_OK;
    RangeLeaves L{};
    for (int c = 0; c < 3; c++) {
        L.rec[c] = rec[c];
        L.len[c] = len[c];
        L.count[c] = count[c];
    }
    const uint64_t blocks = (n + 127) / 128;
    k_range_bytes<<<unsigned(blocks), 128, 0, (cudaStream_t)stream>>>(L, lo, llo, hi, lhi, n, bounds);
    g_cuart_launches += 1;
    return cudaGetLastError() == cudaSuccess ? CUART_OK : CUART_ERR_CUDA;
}
