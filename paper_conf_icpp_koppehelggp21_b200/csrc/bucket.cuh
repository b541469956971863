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

// Histogram layout: [tile group][bucket][tile in group] with groups of kHistGroup
// tiles, so the per-bucket scan reads 32-B runs and a tile's 256 entries share
// sectors with the neighbouring tiles that run at the same time.
constexpr uint64_t kHistGroup = 8;
__device__ __forceinline__ uint64_t hidx(uint32_t b, uint64_t t) {
    return ((t / kHistGroup) * kBuckets + b) * kHistGroup + (t % kHistGroup);
}
__host__ __device__ constexpr uint64_t hist_entries(uint64_t tiles) {
    return ((tiles + kHistGroup - 1) / kHistGroup) * kHistGroup * kBuckets;
}

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
    for (int b = threadIdx.x; b < kBuckets; b += blockDim.x) hist[hidx(b, blockIdx.x)] = h[b];
}

// One CTA per bucket: exclusive scan of its row over the tiles (in place), row total -> totals[b].
__global__ void __launch_bounds__(1024) k_bscan_rows(unsigned int* __restrict__ hist, uint64_t tiles,
                                                     unsigned int* __restrict__ totals) {
    __shared__ unsigned int wsum[32];
    __shared__ unsigned int carry;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    for (uint64_t s0 = 0; s0 < tiles; s0 += blockDim.x) {
        const uint64_t t = s0 + threadIdx.x;
        const unsigned int v = t < tiles ? hist[hidx(blockIdx.x, t)] : 0u;
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
        if (t < tiles) hist[hidx(blockIdx.x, t)] = excl;
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

// Block-wide exclusive scan of one value per thread (kBucketThreads == kBuckets == 256).
__device__ __forceinline__ unsigned int block_excl_scan256(unsigned int v, unsigned int* wtot) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    unsigned int x = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const unsigned int y = __shfl_up_sync(0xffffffffu, x, d);
        if (lane >= d) x += y;
    }
    if (lane == 31) wtot[warp] = x;
    __syncthreads();
    unsigned int before = 0;
#pragma unroll
    for (int w = 0; w < kBucketThreads / 32; w++) before += w < warp ? wtot[w] : 0u;
    return before + x - v;
}

// Tile of kBucketTile queries -> per-bucket runs.  Phase 1: bucket + rank in smem,
// tile-local position jpos[i] (coalesced).  Phase 2: keys staged in smem in bucket
// order; phase 3: each warp copies whole bucket runs to the bucketed batch
// (contiguous source and destination: coalesced reads and writes).
// OPS (update batches): also carry each op's value and original index (its
// priority) to the op's slot; no gather follows, so jpos is not written.
template <class Key, bool OPS = false>
__global__ void __launch_bounds__(kBucketThreads) k_bscatter(const void* __restrict__ q, const uint8_t* __restrict__ lens,
                                                             uint64_t n, uint32_t depth,
                                                             const unsigned int* __restrict__ rowoff,
                                                             const unsigned int* __restrict__ bases,
                                                             void* __restrict__ bq, uint8_t* __restrict__ blens,
                                                             uint16_t* __restrict__ jpos,
                                                             const uint64_t* __restrict__ vals = nullptr,
                                                             uint64_t* __restrict__ bvals = nullptr,
                                                             uint32_t* __restrict__ bidx = nullptr) {
    static_assert(kBucketThreads == kBuckets, "one thread per bucket in the scans");
    constexpr uint32_t KS = Key::kKind == 2 ? 8 : Key::kKind == 1 ? 4 : 32;
    extern __shared__ __align__(16) uint8_t smem[];
    uint8_t* skeys = smem;                                             // kBucketTile * KS
    uint8_t* slens = smem + kBucketTile * KS;                         // kBucketTile (BYTES)
    __shared__ unsigned int h[kBuckets];
    __shared__ unsigned int loc[kBuckets];
    __shared__ unsigned int glb[kBuckets];
    __shared__ unsigned int wtot[kBucketThreads / 32];
    h[threadIdx.x] = 0;
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    uint32_t br[kBucketItems];                                         // bucket << 16 | rank (0xFFFFFFFF = none)
    uint64_t kv[kBucketItems];                                         // integer keys kept in registers
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {                           // all loads first (16 in flight)
        const uint64_t i = base + uint64_t(r) * kBucketThreads + threadIdx.x;
        kv[r] = 0;
        if (i < n && Key::kKind != 3)
            kv[r] = Key::kKind == 2 ? uint64_t(__ldcs((const unsigned long long*)q + i))
                                    : uint64_t(__ldcs((const unsigned int*)q + i));
    }
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint64_t i = base + uint64_t(r) * kBucketThreads + threadIdx.x;
        br[r] = 0xFFFFFFFFu;
        if (i < n) {
            uint32_t b;
            if (Key::kKind == 2) b = bucket_of(KeyU64{kv[r]}, depth);
            else if (Key::kKind == 1) b = bucket_of(KeyU32{uint32_t(kv[r])}, depth);
            else b = bucket_of(Key::template load<false>(q, lens, i), depth);
            br[r] = (b << 16) | atomicAdd(&h[b], 1u);
        }
    }
    __syncthreads();
    const unsigned int mine = h[threadIdx.x];
    loc[threadIdx.x] = block_excl_scan256(mine, wtot);
    glb[threadIdx.x] = bases[threadIdx.x] + rowoff[hidx(threadIdx.x, blockIdx.x)];
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint64_t i = base + uint64_t(r) * kBucketThreads + threadIdx.x;
        if (br[r] != 0xFFFFFFFFu) {
            const uint32_t b = br[r] >> 16, rk = br[r] & 0xFFFFu;
            const uint32_t j = loc[b] + rk;                            // position in the staged tile
            if (Key::kKind == 2) ((uint64_t*)skeys)[j] = kv[r];
            else if (Key::kKind == 1) ((uint32_t*)skeys)[j] = uint32_t(kv[r]);
            else {
                copy_key_to_smem<Key>(q, lens, i, skeys, j);
                slens[j] = lens[i];
            }
            if (OPS) {
                const uint64_t slot = uint64_t(glb[b]) + rk;
                bvals[slot] = __ldcs((const unsigned long long*)vals + i);
                bidx[slot] = uint32_t(i);
            } else {
                jpos[i] = uint16_t(j);
            }
        }
    }
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int b = warp; b < kBuckets; b += kBucketThreads / 32) {
        const uint32_t c = h[b], l0 = loc[b];
        const uint64_t g0 = glb[b];
        for (uint32_t k = lane; k < c; k += 32) {
            if (KS == 8) ((uint64_t*)bq)[g0 + k] = ((const uint64_t*)skeys)[l0 + k];
            else if (KS == 4) ((uint32_t*)bq)[g0 + k] = ((const uint32_t*)skeys)[l0 + k];
            else {
                ((uint4*)bq)[2 * (g0 + k)] = ((const uint4*)skeys)[2 * (l0 + k)];
                ((uint4*)bq)[2 * (g0 + k) + 1] = ((const uint4*)skeys)[2 * (l0 + k) + 1];
                blens[g0 + k] = slens[l0 + k];
            }
        }
    }
}

template <class Key>
constexpr size_t bscatter_smem() {
    return size_t(kBucketTile) * ((Key::kKind == 2 ? 8 : Key::kKind == 1 ? 4 : 32) + (Key::kKind == 3 ? 1 : 0));
}

// Per tile: the tile's results sit in 256 contiguous runs of the bucketed result
// array (one per bucket, located exactly as k_bscatter placed them); each warp
// copies whole runs into shared memory in tile-local order, then
// out[i] = smem[jpos[i]] (coalesced).
__global__ void __launch_bounds__(kBucketThreads) k_bgather(const uint64_t* __restrict__ res,
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

}  // namespace cuart
