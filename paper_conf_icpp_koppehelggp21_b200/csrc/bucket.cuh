// bucket.cuh — K-BUCKET: query pre-bucketing for K-LOOKUP.
//
// P:151 §4.1 batches queries to cut overhead; on B200 the batch can also be
// reordered so that concurrently running warps share subtrees.  The batch is
// partitioned into 256 buckets by the key byte the root branches on (the first
// byte where keys differ, so dense keys with a common prefix still spread), the
// lookup walks the bucketed batch, and a gather restores query order:
//
//   k_bhist      : per-tile (4096 queries) shared-memory histogram -> hist[bucket][tile]
//   k_bscan_rows : one CTA per bucket scans its row over the tiles; k_bscan the totals
//   k_bscatter   : per tile: ranks in shared memory, pos[i] = slot of query i
//                  (written coalesced), keys staged in smem in bucket order and
//                  written as contiguous runs -> tile-stable bucketed batch
//   (k_lookup over the bucketed keys, results in bucketed order)
//   k_bgather    : out[i] = res[pos[i]]
//
// While the lookups of one bucket run, the working set is that bucket's slice of
// the tree (c3: ~10 MB of nodes/leaves per bucket), i.e. L2-resident, instead of
// random lines over the whole 2.5 GB index.  Because slots follow tile order, the
// gather walks every bucket's run front to back (256 live lines), so the reordering
// costs streaming traffic only (~45 B/query).
#pragma once
#include "kernels.cuh"

namespace cuart {

constexpr int kBucketBits = 8;
constexpr int kBuckets = 1 << kBucketBits;
constexpr int kBucketThreads = 256;
constexpr int kBucketItems = 16;
constexpr int kBucketTile = kBucketThreads * kBucketItems;

template <class Key>
__device__ __forceinline__ uint32_t bucket_of(const Key& k, uint32_t depth) {
    return depth < k.len() ? k.byte(depth) : 0u;
}

// Per-tile histogram, stored bucket-major: hist[b * tiles + t].
template <class Key>
__global__ void __launch_bounds__(kBucketThreads) k_bhist(const void* __restrict__ q, const uint8_t* __restrict__ lens,
                                                          uint64_t n, uint32_t depth, unsigned int* __restrict__ hist) {
    __shared__ unsigned int h[kBuckets];
    for (int b = threadIdx.x; b < kBuckets; b += blockDim.x) h[b] = 0;
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    for (int r = 0; r < kBucketItems; r++) {
        const uint64_t i = base + uint64_t(r) * kBucketThreads + threadIdx.x;
        if (i < n) atomicAdd(&h[bucket_of(Key::template load<true>(q, lens, i), depth)], 1u);
    }
    __syncthreads();
    for (int b = threadIdx.x; b < kBuckets; b += blockDim.x) hist[uint64_t(b) * gridDim.x + blockIdx.x] = h[b];
}

// One CTA per bucket: exclusive scan of its row over the tiles (in place), row total -> totals[b].
__global__ void __launch_bounds__(1024) k_bscan_rows(unsigned int* __restrict__ hist, uint64_t tiles,
                                                     unsigned int* __restrict__ totals) {
    __shared__ unsigned int wsum[32];
    __shared__ unsigned int carry;
    unsigned int* row = hist + uint64_t(blockIdx.x) * tiles;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    for (uint64_t s0 = 0; s0 < tiles; s0 += blockDim.x) {
        const uint64_t t = s0 + threadIdx.x;
        const unsigned int v = t < tiles ? row[t] : 0u;
        unsigned int x = v;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const unsigned int y = __shfl_up_sync(0xffffffffu, x, d);
            if (lane >= d) x += y;
        }
        if (lane == 31) wsum[warp] = x;
        __syncthreads();
        if (warp == 0) {
            unsigned int w = wsum[lane];
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const unsigned int y = __shfl_up_sync(0xffffffffu, w, d);
                if (lane >= d) w += y;
            }
            wsum[lane] = w;
        }
        __syncthreads();
        const unsigned int excl = carry + (warp ? wsum[warp - 1] : 0u) + x - v;
        if (t < tiles) row[t] = excl;
        __syncthreads();
        if (threadIdx.x == blockDim.x - 1) carry = excl + v;
        __syncthreads();
    }
    if (threadIdx.x == 0) totals[blockIdx.x] = carry;
}

// totals -> exclusive bucket bases (in place), one CTA of kBuckets threads
__global__ void __launch_bounds__(kBuckets) k_bscan(unsigned int* __restrict__ counts) {
    __shared__ unsigned int s[kBuckets];
    const int t = threadIdx.x;
    s[t] = counts[t];
    __syncthreads();
    for (int d = 1; d < kBuckets; d <<= 1) {
        const unsigned int v = t >= d ? s[t - d] : 0u;
        __syncthreads();
        s[t] += v;
        __syncthreads();
    }
    counts[t] = s[t] - counts[t];   // exclusive
}

template <class Key>
__device__ __forceinline__ void copy_key_to_smem(const void* q, const uint8_t* lens, uint64_t i, uint8_t* sm, uint32_t j) {
    if (Key::kKind == 2) ((uint64_t*)sm)[j] = __ldcs((const unsigned long long*)q + i);
    else if (Key::kKind == 1) ((uint32_t*)sm)[j] = __ldcs((const unsigned int*)q + i);
    else {
        const uint4* s = (const uint4*)q + 2 * i;
        uint4* d = (uint4*)sm + 2 * j;
        d[0] = __ldcs(s);
        d[1] = __ldcs(s + 1);
    }
}

// Tile of kBucketTile queries -> per-bucket runs.  Phase 1: bucket + rank in smem,
// pos[i] written coalesced.  Phase 2: keys staged in smem in bucket order, then
// written out with consecutive threads on consecutive slots of a run.
template <class Key>
__global__ void __launch_bounds__(kBucketThreads) k_bscatter(const void* __restrict__ q, const uint8_t* __restrict__ lens,
                                                             uint64_t n, uint32_t depth,
                                                             const unsigned int* __restrict__ rowoff,
                                                             const unsigned int* __restrict__ bases,
                                                             void* __restrict__ bq, uint8_t* __restrict__ blens,
                                                             uint16_t* __restrict__ jpos) {
    constexpr uint32_t KS = Key::kKind == 2 ? 8 : Key::kKind == 1 ? 4 : 32;
    extern __shared__ __align__(16) uint8_t smem[];
    uint8_t* skeys = smem;                                             // kBucketTile * KS
    uint32_t* sslot = (uint32_t*)(smem + kBucketTile * KS);           // kBucketTile
    uint8_t* slens = (uint8_t*)(sslot + kBucketTile);                 // kBucketTile (BYTES)
    __shared__ unsigned int h[kBuckets];
    __shared__ unsigned int loc[kBuckets];
    __shared__ unsigned int glb[kBuckets];
    for (int b = threadIdx.x; b < kBuckets; b += blockDim.x) h[b] = 0;
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    uint32_t bk[kBucketItems], rk[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint64_t i = base + uint64_t(r) * kBucketThreads + threadIdx.x;
        bk[r] = kBuckets;
        if (i < n) {
            bk[r] = bucket_of(Key::template load<false>(q, lens, i), depth);
            rk[r] = atomicAdd(&h[bk[r]], 1u);
        }
    }
    __syncthreads();
    if (threadIdx.x < kBuckets) {                                      // local exclusive offsets (serial scan, 256)
        glb[threadIdx.x] = bases[threadIdx.x] + rowoff[uint64_t(threadIdx.x) * gridDim.x + blockIdx.x];
    }
    if (threadIdx.x == 0) {
        unsigned int acc = 0;
        for (int b = 0; b < kBuckets; b++) {
            loc[b] = acc;
            acc += h[b];
        }
    }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint64_t i = base + uint64_t(r) * kBucketThreads + threadIdx.x;
        if (bk[r] < uint32_t(kBuckets)) {
            const uint32_t j = loc[bk[r]] + rk[r];                     // position in the staged tile
            const uint32_t slot = glb[bk[r]] + rk[r];                  // position in the bucketed batch
            copy_key_to_smem<Key>(q, lens, i, skeys, j);
            if (Key::kKind == 3) slens[j] = lens[i];
            sslot[j] = slot;
            jpos[i] = uint16_t(j);                                     // tile-local position (coalesced)
        }
    }
    __syncthreads();
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    for (uint32_t j = threadIdx.x; j < cnt; j += blockDim.x) {
        const uint32_t slot = sslot[j];
        if (KS == 8) ((uint64_t*)bq)[slot] = ((const uint64_t*)skeys)[j];
        else if (KS == 4) ((uint32_t*)bq)[slot] = ((const uint32_t*)skeys)[j];
        else {
            ((uint4*)bq)[2 * uint64_t(slot)] = ((const uint4*)skeys)[2 * j];
            ((uint4*)bq)[2 * uint64_t(slot) + 1] = ((const uint4*)skeys)[2 * j + 1];
            blens[slot] = slens[j];
        }
    }
}

template <class Key>
constexpr size_t bscatter_smem() {
    return size_t(kBucketTile) * ((Key::kKind == 2 ? 8 : Key::kKind == 1 ? 4 : 32) + 4 + (Key::kKind == 3 ? 1 : 0));
}

// Per tile: the tile's results sit in 256 contiguous runs of the bucketed result
// array (one per bucket, located exactly as k_bscatter placed them); load them in
// tile-local order into shared memory, then out[i] = smem[jpos[i]] (coalesced).
__global__ void __launch_bounds__(kBucketThreads) k_bgather(const uint64_t* __restrict__ res,
                                                            const uint16_t* __restrict__ jpos, uint64_t n,
                                                            const unsigned int* __restrict__ rowoff,
                                                            const unsigned int* __restrict__ bases,
                                                            uint64_t* __restrict__ out) {
    __shared__ uint64_t sres[kBucketTile];
    __shared__ unsigned int loc[kBuckets + 1];
    __shared__ unsigned int glb[kBuckets];
    const uint64_t t = blockIdx.x, tiles = gridDim.x;
    const uint64_t base = t * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    if (threadIdx.x < kBuckets) {
        const int b = threadIdx.x;
        const unsigned int off = rowoff[uint64_t(b) * tiles + t];
        const unsigned int btotal = (b + 1 < kBuckets ? bases[b + 1] : unsigned(n)) - bases[b];
        const unsigned int next = t + 1 < tiles ? rowoff[uint64_t(b) * tiles + t + 1] : btotal;
        glb[b] = bases[b] + off;
        loc[b + 1] = next - off;                                        // this tile's count in bucket b
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned int acc = 0;
        loc[0] = 0;
        for (int b = 0; b < kBuckets; b++) {
            acc += loc[b + 1];
            loc[b + 1] = acc;
        }
    }
    __syncthreads();
    for (uint32_t j = threadIdx.x; j < cnt; j += blockDim.x) {
        uint32_t lo = 0, hi = kBuckets;                                 // bucket b with loc[b] <= j < loc[b+1]
        while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (loc[mid] <= j) lo = mid;
            else hi = mid;
        }
        sres[j] = __ldcs((const unsigned long long*)res + glb[lo] + (j - loc[lo]));
    }
    __syncthreads();
    for (uint32_t k = threadIdx.x; k < cnt; k += blockDim.x)
        __stcs((unsigned long long*)out + base + k, (unsigned long long)sres[__ldcs(jpos + base + k)]);
}

}  // namespace cuart
