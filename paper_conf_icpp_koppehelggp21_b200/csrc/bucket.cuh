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
//
// All three streaming kernels are HBM-bound: every global load of a tile is issued
// before its first use (16 per thread in flight), and every store instruction is a
// full warp writing consecutive addresses.
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

// `depth` packs the key byte the buckets are taken from (bits 7..0: the root's
// branch depth) and a right shift of that byte (bits 15..8): shift s gives 256 >> s
// buckets (the upper bucket ids stay empty; every kernel below is unchanged).
template <class Key>
__device__ __forceinline__ uint32_t bucket_of(const Key& k, uint32_t depth) {
    const uint32_t d = depth & 0xFFu;
    return d < k.len() ? k.byte(d) >> (depth >> 8) : 0u;
}

// Bucket of query i straight from the batch: integer keys from their word, byte
// strings from their length and the single key byte the bucket needs.
template <class Key>
__device__ __forceinline__ uint32_t bucket_at(const void* q, const uint8_t* lens, uint64_t i, uint32_t depth) {
    if (Key::kKind == 2) return bucket_of(KeyU64{uint64_t(__ldcs((const unsigned long long*)q + i))}, depth);
    if (Key::kKind == 1) return bucket_of(KeyU32{uint32_t(__ldcs((const unsigned int*)q + i))}, depth);
    const uint32_t l = __ldcs(lens + i), d = depth & 0xFFu;
    return d < l ? uint32_t(__ldcs((const uint8_t*)q + 32 * i + d)) >> (depth >> 8) : 0u;
}

// Part functions of the K-BUCKET kernels.  ByteBucket: the single-GPU bucket (root
// branch byte >> shift, packed in `depth` as above).  OwnerPart (multi-GPU, §8(e)):
// K-ROUTE fused with K-BUCKET -- part = owner << lbpo | (the owner's root branch
// byte >> (8 - lbpo)), owner = number of splitters <= the key's first 8 bytes read
// big-endian.  Parts are numbered owner-major, so the bucketed batch is also the
// routed batch: owner o's ops are one contiguous run of the send order, already
// bucketed for o's walk.
struct ByteBucket {
    static constexpr bool kFilter = false;
    uint32_t depth;
    __host__ __device__ ByteBucket(uint32_t d = 0) : depth(d) {}
    __device__ __forceinline__ bool skip(uint64_t) const { return false; }
    template <class Key>
    __device__ __forceinline__ uint32_t of(const Key& k) const { return bucket_of(k, depth); }
    template <class Key>
    __device__ __forceinline__ uint32_t at(const void* q, const uint8_t* lens, uint64_t i) const {
        return bucket_at<Key>(q, lens, i, depth);
    }
};

template <class Key>
__device__ __forceinline__ uint64_t key_prefix8(const Key& k) {
    if (Key::kKind == 2) return uint64_t(((const KeyU64&)k).k);
    if (Key::kKind == 1) return uint64_t(((const KeyU32&)k).k) << 32;
    return bswap64(((const KeyBytes&)k).w[0]);                 // zero-padded past the length
}

struct OwnerPart {
    static constexpr bool kFilter = false;
    uint32_t nsp;                      // number of splitters (ranks - 1)
    uint32_t lbpo;                     // bucket bits per owner
    uint64_t sp[kMaxSeg - 1];          // ascending splitters over the 8-byte prefix
    uint8_t depth[kMaxSeg];            // every owner's root branch depth
    __device__ __forceinline__ bool skip(uint64_t) const { return false; }
    template <class Key>
    __device__ __forceinline__ uint32_t owner(const Key& k) const {
        const uint64_t p = key_prefix8(k);
        uint32_t o = 0;
#pragma unroll 1
        for (uint32_t j = 0; j < nsp; j++) o += sp[j] <= p ? 1u : 0u;
        return o;
    }
    template <class Key>
    __device__ __forceinline__ uint32_t of(const Key& k) const {
        const uint32_t o = owner(k);
        const uint32_t d = depth[o];
        const uint32_t b = d < k.len() ? k.byte(d) : 0u;
        return (o << lbpo) | (b >> (8 - lbpo));
    }
    template <class Key>
    __device__ __forceinline__ uint32_t at(const void* q, const uint8_t* lens, uint64_t i) const {
        return of(Key::template load<true>(q, lens, i));
    }
};

// OwnerPart over one kind of op of a mixed batch (config 5's rounds, reading C7):
// ops whose flag differs from `want` are skipped -- not counted, not staged, and a
// skipped lookup's jpos is kSkipPos, for which the gather writes CUART_MISS.  One
// pass per kind replaces the stable partition of the batch and its inverse.
struct FilteredOwnerPart : OwnerPart {
    static constexpr bool kFilter = true;
    const uint8_t* flags;
    uint32_t want;
    __device__ __forceinline__ bool skip(uint64_t i) const { return (__ldcs(flags + i) != 0) != (want != 0); }
};
constexpr uint16_t kSkipPos = 0xFFFF;

// Fused push of the multi-GPU exchange (transport p2p): the staged runs of k_bscatter
// are stored straight into the receive windows of their owners (peer memory mapped
// over NVLink / NVSwitch): send-order slot d of a part of owner o lands at
// keys[o] + d + adj[o] (adj = this source's first slot in o's window minus o's first
// send-order slot).  nrep > 0 (replica mode): every op goes to all nrep windows.
struct PushDst {
    void* keys[kMaxSeg];
    uint8_t* lens[kMaxSeg];
    uint64_t* vals[kMaxSeg];
    uint32_t* prio[kMaxSeg];
    const long long* adj;              // device, per owner (written by the count exchange)
    uint32_t lbpo;
    uint32_t nrep;
};

#ifndef CUART_SCATTER_MIN_BLOCKS
#define CUART_SCATTER_MIN_BLOCKS 1
#endif
constexpr int kScatterMinBlocks = CUART_SCATTER_MIN_BLOCKS;   // register cap of the lookup scatter (A/B knob)
#ifndef CUART_HIST_MIN_BLOCKS
#define CUART_HIST_MIN_BLOCKS 1
#endif
constexpr int kHistMinBlocks = CUART_HIST_MIN_BLOCKS;

// Block-wide exclusive scan of one value per thread (kBucketThreads == kBuckets == 256).
// Contains one __syncthreads; the caller syncs before reusing wtot.
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

// Per-tile histogram, stored bucket-major: hist[hidx(b, t)].  Every key of the tile
// is loaded before the first shared-memory atomic; with VEC (queries 16-B aligned)
// integer keys arrive in 16-B loads (2 u64 / 4 u32 keys per load): 1.27 ms per
// 2^30 u64 keys (6.8 TB/s) against 2.08 ms with 8-B loads (tools/bucket_micro.cu).
template <class Key, bool VEC, class PF = ByteBucket>
__global__ void __launch_bounds__(kBucketThreads, kHistMinBlocks) k_bhist(const void* __restrict__ q, const uint8_t* __restrict__ lens,
                                                          uint64_t n, PF pf, unsigned int* __restrict__ hist) {
    __shared__ unsigned int h[kBuckets];
    h[threadIdx.x] = 0;
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    if (VEC && Key::kKind != 3) {
        constexpr int PER = Key::kKind == 2 ? 2 : 4;                  // keys per 16-B load
        constexpr int LOADS = kBucketItems / PER;
        uint4 v[LOADS];
#pragma unroll
        for (int r = 0; r < LOADS; r++) {
            const uint64_t i = base + uint64_t(PER) * (uint64_t(r) * kBucketThreads + threadIdx.x);
            v[r] = i + PER <= n ? __ldcs((const uint4*)((const uint8_t*)q + i * (Key::kKind == 2 ? 8 : 4)))
                                : make_uint4(0, 0, 0, 0);
        }
#pragma unroll
        for (int r = 0; r < LOADS; r++) {
            const uint64_t i = base + uint64_t(PER) * (uint64_t(r) * kBucketThreads + threadIdx.x);
            if (i + PER <= n) {
                if (Key::kKind == 2) {
                    if (!pf.skip(i)) atomicAdd(&h[pf.of(KeyU64{uint64_t(v[r].x) | (uint64_t(v[r].y) << 32)})], 1u);
                    if (!pf.skip(i + 1)) atomicAdd(&h[pf.of(KeyU64{uint64_t(v[r].z) | (uint64_t(v[r].w) << 32)})], 1u);
                } else {
                    if (!pf.skip(i)) atomicAdd(&h[pf.of(KeyU32{v[r].x})], 1u);
                    if (!pf.skip(i + 1)) atomicAdd(&h[pf.of(KeyU32{v[r].y})], 1u);
                    if (!pf.skip(i + 2)) atomicAdd(&h[pf.of(KeyU32{v[r].z})], 1u);
                    if (!pf.skip(i + 3)) atomicAdd(&h[pf.of(KeyU32{v[r].w})], 1u);
                }
            } else {
                for (uint64_t e = i; e < n && e < i + PER; e++)
                    if (!pf.skip(e)) atomicAdd(&h[pf.template at<Key>(q, lens, e)], 1u);
            }
        }
    } else {
        uint32_t bk[kBucketItems];
#pragma unroll
        for (int r = 0; r < kBucketItems; r++) {
            const uint64_t i = base + uint64_t(r) * kBucketThreads + threadIdx.x;
            bk[r] = i < n && !pf.skip(i) ? pf.template at<Key>(q, lens, i) : 0xFFFFFFFFu;
        }
#pragma unroll
        for (int r = 0; r < kBucketItems; r++)
            if (bk[r] != 0xFFFFFFFFu) atomicAdd(&h[bk[r]], 1u);
    }
    __syncthreads();
    hist[hidx(threadIdx.x, blockIdx.x)] = h[threadIdx.x];
}

// One CTA per bucket: exclusive scan of its row over the tiles (in place), row
// total -> totals[b].  A hist group is kHistGroup = 8 consecutive tiles of this
// bucket = one 32-B sector.
static __global__ void __launch_bounds__(kBucketThreads) k_bscan_rows(unsigned int* __restrict__ hist, uint64_t tiles,
                                                               unsigned int* __restrict__ totals) {
    static_assert(kHistGroup == 8, "one 32-B sector per thread");
    __shared__ unsigned int wtot[kBucketThreads / 32];
    __shared__ unsigned int pass_total;
    const uint32_t b = blockIdx.x;
    const uint64_t groups = (tiles + kHistGroup - 1) / kHistGroup;
    // a thread owns GPT consecutive hist groups per pass (GPT x 32 B in flight), so
    // one pass covers 256 x GPT x 8 tiles
    constexpr int GPT = 4;
    unsigned int carry = 0;
    for (uint64_t g0 = 0; g0 < groups; g0 += uint64_t(kBucketThreads) * GPT) {
        unsigned int v[GPT][8];
#pragma unroll
        for (int u = 0; u < GPT; u++) {
            const uint64_t g = g0 + uint64_t(threadIdx.x) * GPT + u;
#pragma unroll
            for (int k = 0; k < 8; k++) v[u][k] = 0;
            if (g < groups) {
                const uint4* p = (const uint4*)(hist + (g * kBuckets + b) * kHistGroup);
                const uint4 a = p[0], c = p[1];
                v[u][0] = a.x; v[u][1] = a.y; v[u][2] = a.z; v[u][3] = a.w;
                v[u][4] = c.x; v[u][5] = c.y; v[u][6] = c.z; v[u][7] = c.w;
#pragma unroll
                for (int k = 0; k < 8; k++)
                    if (g * kHistGroup + k >= tiles) v[u][k] = 0;   // padding entries are never written by k_bhist
            }
        }
        unsigned int s = 0;
#pragma unroll
        for (int u = 0; u < GPT; u++)
#pragma unroll
            for (int k = 0; k < 8; k++) s += v[u][k];
        const unsigned int ex = block_excl_scan256(s, wtot);
        unsigned int run = carry + ex;
#pragma unroll
        for (int u = 0; u < GPT; u++) {
            const uint64_t g = g0 + uint64_t(threadIdx.x) * GPT + u;
            unsigned int o[8];
#pragma unroll
            for (int k = 0; k < 8; k++) {
                o[k] = run;
                run += v[u][k];
            }
            if (g < groups) {
                uint4* p = (uint4*)(hist + (g * kBuckets + b) * kHistGroup);
                p[0] = make_uint4(o[0], o[1], o[2], o[3]);
                p[1] = make_uint4(o[4], o[5], o[6], o[7]);
            }
        }
        if (threadIdx.x == kBucketThreads - 1) pass_total = ex + s;
        __syncthreads();
        carry += pass_total;
        __syncthreads();                                          // wtot / pass_total are reused next pass
    }
    if (threadIdx.x == 0) totals[b] = carry;
}

// totals -> exclusive bucket bases (in place), one CTA of kBuckets threads, and the
// grand total at counts[kBuckets] (so counts needs kBuckets + 1 entries).
// Only the first nb buckets are in use (256 >> shift): the others count 0 (their
// totals were never written) and get base = n.
static __global__ void __launch_bounds__(kBuckets) k_bscan(unsigned int* __restrict__ counts, uint32_t nb) {
    __shared__ unsigned int s[kBuckets];
    const int t = threadIdx.x;
    const unsigned int own = uint32_t(t) < nb ? counts[t] : 0u;
    s[t] = own;
    __syncthreads();
    for (int d = 1; d < kBuckets; d <<= 1) {
        const unsigned int v = t >= d ? s[t - d] : 0u;
        __syncthreads();
        s[t] += v;
        __syncthreads();
    }
    counts[t] = s[t] - own;   // exclusive
    if (t == kBuckets - 1) counts[kBuckets] = s[t];
}

template <class Key>
__device__ __forceinline__ void copy_key_to_smem(const void* q, uint64_t i, uint8_t* sm, uint32_t j) {
    if (Key::kKind == 2) ((uint64_t*)sm)[j] = __ldcs((const unsigned long long*)q + i);
    else if (Key::kKind == 1) ((uint32_t*)sm)[j] = __ldcs((const unsigned int*)q + i);
    else {
        const uint4* s = (const uint4*)q + 2 * i;
        uint4* d = (uint4*)sm + 2 * j;
        d[0] = __ldcs(s);
        d[1] = __ldcs(s + 1);
    }
}

// Tile of kBucketTile queries -> per-bucket runs.  Phase 1: all keys (and, for
// update batches, values) loaded into registers, bucket + rank in shared memory.
// Phase 2: staged in shared memory in bucket order together with the bucket of
// every staged position (and the tile-local op index for updates); jpos[i] =
// staged position of query i (coalesced).  Phase 3: thread-per-position copy of
// the staged tile to the bucketed batch — consecutive threads write consecutive
// slots of a bucket run, so every store instruction is a full warp and a thread
// has 16 independent stores.
// OPS (update batches): each op's value and original index (its priority)
// travel with it; no gather follows, so jpos is not written.
// prio_base (OPS): the priority written with an op is prio_base + its index in the
// batch (the multi-GPU layer numbers ops globally, rank-major, reading C7).
// PUSH: the runs go to the owners' receive windows (PushDst), not to bq/blens/bvals/bidx.
template <class Key, bool OPS = false, class PF = ByteBucket, bool PUSH = false>
__global__ void __launch_bounds__(kBucketThreads, !OPS && Key::kKind != 3 ? kScatterMinBlocks : 1) k_bscatter(const void* __restrict__ q, const uint8_t* __restrict__ lens,
                                                             uint64_t n, PF pf,
                                                             const unsigned int* __restrict__ rowoff,
                                                             const unsigned int* __restrict__ bases,
                                                             void* __restrict__ bq, uint8_t* __restrict__ blens,
                                                             uint16_t* __restrict__ jpos,
                                                             const uint64_t* __restrict__ vals = nullptr,
                                                             uint64_t* __restrict__ bvals = nullptr,
                                                             uint32_t* __restrict__ bidx = nullptr,
                                                             uint32_t prio_base = 0, PushDst pd = PushDst{}) {
    static_assert(kBucketThreads == kBuckets, "one thread per bucket in the scans");
    constexpr uint32_t KS = Key::kKind == 2 ? 8 : Key::kKind == 1 ? 4 : 32;
    extern __shared__ __align__(16) uint8_t smem[];
    uint8_t* skeys = smem;                                                      // kBucketTile * KS
    uint64_t* svals = (uint64_t*)(smem + kBucketTile * KS);                     // OPS: kBucketTile * 8
    uint16_t* sidx = (uint16_t*)(smem + kBucketTile * (KS + (OPS ? 8 : 0)));   // OPS: kBucketTile * 2
    uint8_t* sb = smem + kBucketTile * (KS + (OPS ? 10 : 0));                   // bucket of each staged position
    uint8_t* slens = sb + kBucketTile;                                          // BYTES: kBucketTile
    __shared__ unsigned int h[kBuckets];
    __shared__ unsigned int loc[kBuckets];
    __shared__ unsigned int glb[kBuckets];
    __shared__ unsigned int wtot[kBucketThreads / 32];
    __shared__ long long padj[PUSH ? kBuckets : 1];                   // PUSH: per-part window adjustment
    __shared__ void* swin[PUSH ? 4 * kMaxSeg : 1];                     // PUSH: keys / lens / vals / prio windows
    h[threadIdx.x] = 0;
    const unsigned int gb = bases[threadIdx.x] + rowoff[hidx(threadIdx.x, blockIdx.x)];   // issued first
    if (PUSH) {
        if (pd.nrep == 0) padj[threadIdx.x] = pd.adj[threadIdx.x >> pd.lbpo < kMaxSeg ? threadIdx.x >> pd.lbpo : 0];
        if (threadIdx.x < kMaxSeg) {
            swin[threadIdx.x] = pd.keys[threadIdx.x];
            swin[kMaxSeg + threadIdx.x] = pd.lens[threadIdx.x];
            swin[2 * kMaxSeg + threadIdx.x] = pd.vals[threadIdx.x];
            swin[3 * kMaxSeg + threadIdx.x] = pd.prio[threadIdx.x];
            if (pd.nrep) padj[threadIdx.x] = threadIdx.x < pd.nrep ? pd.adj[threadIdx.x] : 0;
        }
    }
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    __shared__ unsigned int staged_n;                                  // ops staged (all of them unless filtered)
    uint32_t scnt = cnt;
    __syncthreads();
    uint32_t br[kBucketItems];                                         // bucket << 16 | rank (0xFFFFFFFF = none)
    uint64_t kv[kBucketItems];                                         // integer keys kept in registers
    uint64_t vv[OPS ? kBucketItems : 1];                               // update values kept in registers
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {                           // all loads first
        const uint32_t j = uint32_t(r) * kBucketThreads + threadIdx.x;
        kv[r] = 0;
        if (j < cnt && Key::kKind != 3)
            kv[r] = Key::kKind == 2 ? uint64_t(__ldcs((const unsigned long long*)q + base + j))
                                    : uint64_t(__ldcs((const unsigned int*)q + base + j));
        if (OPS) vv[OPS ? r : 0] = j < cnt ? uint64_t(__ldcs((const unsigned long long*)vals + base + j)) : 0ull;
    }
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * kBucketThreads + threadIdx.x;
        br[r] = 0xFFFFFFFFu;
        if (j < cnt && !pf.skip(base + j)) {
            uint32_t b;
            if (Key::kKind == 2) b = pf.of(KeyU64{kv[r]});
            else if (Key::kKind == 1) b = pf.of(KeyU32{uint32_t(kv[r])});
            else b = pf.template at<Key>(q, lens, base + j);
            br[r] = (b << 16) | atomicAdd(&h[b], 1u);
        }
    }
    __syncthreads();
    const unsigned int mine = h[threadIdx.x];
    const unsigned int lb = block_excl_scan256(mine, wtot);
    loc[threadIdx.x] = lb;
    glb[threadIdx.x] = gb - lb;                                        // slot = glb[b] + staged position (mod 2^32)
    if (threadIdx.x == kBucketThreads - 1) staged_n = lb + mine;
    __syncthreads();
    scnt = PF::kFilter ? staged_n : cnt;
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t jt = uint32_t(r) * kBucketThreads + threadIdx.x;   // tile-local op position
        if (PF::kFilter && !OPS && br[r] == 0xFFFFFFFFu && jt < cnt)
            __stcs((unsigned short*)jpos + base + jt, (unsigned short)kSkipPos);
        if (br[r] != 0xFFFFFFFFu) {
            const uint32_t b = br[r] >> 16, rk = br[r] & 0xFFFFu;
            const uint32_t j = loc[b] + rk;                            // position in the staged tile
            sb[j] = uint8_t(b);
            if (Key::kKind == 2) ((uint64_t*)skeys)[j] = kv[r];
            else if (Key::kKind == 1) ((uint32_t*)skeys)[j] = uint32_t(kv[r]);
            else {
                copy_key_to_smem<Key>(q, base + jt, skeys, j);
                slens[j] = lens[base + jt];
            }
            if (OPS) {
                svals[j] = vv[OPS ? r : 0];
                sidx[j] = uint16_t(jt);
            } else {
                __stcs((unsigned short*)jpos + base + jt, (unsigned short)j);
            }
        }
    }
    __syncthreads();
    if (PUSH) {                                                        // fused route: runs -> owner windows
#pragma unroll 4
        for (int r = 0; r < kBucketItems; r++) {
            const uint32_t j = uint32_t(r) * kBucketThreads + threadIdx.x;
            if (j >= scnt) continue;
            const uint32_t b = sb[j];
            const uint64_t dsend = uint64_t(glb[b] + j);                  // send-order slot
            const uint32_t w0 = pd.nrep ? 0u : (b >> pd.lbpo), w1 = pd.nrep ? pd.nrep : w0 + 1;
            for (uint32_t w = w0; w < w1; w++) {
                const uint64_t dst = dsend + uint64_t(padj[pd.nrep ? w : b]);
                void* kw = swin[w];
                if (KS == 8) __stcs((unsigned long long*)kw + dst, (unsigned long long)((const uint64_t*)skeys)[j]);
                else if (KS == 4) __stcs((unsigned int*)kw + dst, ((const uint32_t*)skeys)[j]);
                else {
                    __stcs((uint4*)kw + 2 * dst, ((const uint4*)skeys)[2 * j]);
                    __stcs((uint4*)kw + 2 * dst + 1, ((const uint4*)skeys)[2 * j + 1]);
                    ((uint8_t*)swin[kMaxSeg + w])[dst] = slens[j];
                }
                if (OPS) {
                    __stcs((unsigned long long*)swin[2 * kMaxSeg + w] + dst, (unsigned long long)svals[j]);
                    __stcs((unsigned int*)swin[3 * kMaxSeg + w] + dst, unsigned(prio_base + base + sidx[j]));
                }
            }
        }
        return;
    }
#pragma unroll 4
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * kBucketThreads + threadIdx.x;
        if (j < scnt) {
            const uint64_t dst = uint64_t(glb[sb[j]] + j);                // n < 2^32: exact
            if (KS == 8) __stcs((unsigned long long*)bq + dst, (unsigned long long)((const uint64_t*)skeys)[j]);
            else if (KS == 4) __stcs((unsigned int*)bq + dst, ((const uint32_t*)skeys)[j]);
            else {
                __stcs((uint4*)bq + 2 * dst, ((const uint4*)skeys)[2 * j]);
                __stcs((uint4*)bq + 2 * dst + 1, ((const uint4*)skeys)[2 * j + 1]);
                blens[dst] = slens[j];
            }
            if (OPS) {
                __stcs((unsigned long long*)bvals + dst, (unsigned long long)svals[j]);
                __stcs((unsigned int*)bidx + dst, unsigned(prio_base + base + sidx[j]));
            }
        }
    }
}

template <class Key, bool OPS = false>
constexpr size_t bscatter_smem() {
    return size_t(kBucketTile) *
           ((Key::kKind == 2 ? 8 : Key::kKind == 1 ? 4 : 32) + (OPS ? 10 : 0) + 1 + (Key::kKind == 3 ? 1 : 0));
}

__device__ __forceinline__ void cp_async8(void* smem, const void* g) {
    const unsigned sa = unsigned(__cvta_generic_to_shared(smem));
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(sa), "l"(g));
}
__device__ __forceinline__ void cp_async_wait_all() {
    asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
}

#ifndef CUART_GATHER_MIN_BLOCKS
#define CUART_GATHER_MIN_BLOCKS 5
#endif
// 5 CTAs/SM: <= 51 registers instead of 63, occupancy 62% instead of 50%; measured
// c3 gather 3.79 -> 3.54 ms per 2^30 (profiles/r02/ab_scatter_gather.txt)
constexpr int kGatherMinBlocks = CUART_GATHER_MIN_BLOCKS;

// Per tile: the tile's results sit in 256 contiguous runs of the bucketed result
// array (one per bucket, located exactly as k_bscatter placed them).  The run
// offsets and jpos are loaded first; the runs are copied thread-per-position into
// shared memory with cp.async (no registers held across the DRAM round trip: 3.77
// ms per 2^30 against 4.19 ms with register staging, tools/bucket_micro.cu), then
// out[i] = smem[jpos[i]] (coalesced).
// SEG: out is ignored and result i goes to so.at(i) (fused return to the requesting GPUs).
// FILT: the batch was bucketed with a filtered part function: only nkept of its n ops
// were staged; a skipped op (jpos == kSkipPos) gets CUART_MISS.
template <bool SEG = false, bool FILT = false>
__global__ void __launch_bounds__(kBucketThreads, kGatherMinBlocks) k_bgather(const uint64_t* __restrict__ res,
                                                            const uint16_t* __restrict__ jpos, uint64_t n,
                                                            const unsigned int* __restrict__ rowoff,
                                                            const unsigned int* __restrict__ bases,
                                                            uint64_t* __restrict__ out, SegOut so = SegOut{},
                                                            uint64_t nkept = 0) {
    __shared__ uint64_t sres[kBucketTile];
    __shared__ uint8_t bof[kBucketTile];                               // bucket of each staged position
    __shared__ unsigned int loc[kBuckets];
    __shared__ unsigned int glb[kBuckets];
    __shared__ unsigned int wtot[kBucketThreads / 32];
    const uint64_t t = blockIdx.x, tiles = gridDim.x;
    const uint64_t base = t * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    const int b = threadIdx.x;
    const unsigned int off = rowoff[hidx(b, t)];
    const unsigned int bb = bases[b];
    const unsigned int bnext = b + 1 < kBuckets ? bases[b + 1] : unsigned(FILT ? nkept : n);
    const unsigned int next = t + 1 < tiles ? rowoff[hidx(b, t + 1)] : bnext - bb;
    uint16_t jp[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t k = uint32_t(r) * kBucketThreads + threadIdx.x;
        jp[r] = k < cnt ? __ldcs(jpos + base + k) : 0;
    }
    const unsigned int c_b = next - off;
    glb[b] = bb + off;
    const unsigned int l_b = block_excl_scan256(c_b, wtot);
    loc[b] = l_b;
    for (unsigned int k = 0; k < c_b; k++) bof[l_b + k] = uint8_t(b);
    __shared__ unsigned int staged_n;
    if (FILT && b == kBuckets - 1) staged_n = l_b + c_b;
    __syncthreads();
    const uint32_t scnt = FILT ? staged_n : cnt;
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = uint32_t(r) * kBucketThreads + threadIdx.x;
        if (j < scnt) {
            const uint32_t bj = bof[j];
            cp_async8(&sres[j], res + glb[bj] + (j - loc[bj]));
        }
    }
    cp_async_wait_all();
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t k = uint32_t(r) * kBucketThreads + threadIdx.x;
        if (k < cnt) {
            unsigned long long* dst = SEG ? (unsigned long long*)so.at(base + k) : (unsigned long long*)out + base + k;
            __stcs(dst, FILT && jp[r] == kSkipPos ? ~0ull : (unsigned long long)sres[jp[r]]);
        }
    }
}

// ============================================================================ tile form
// K-BUCKET without a global scatter.  The global form above needs every tile's
// per-bucket counts before any key moves (k_bhist reads the whole batch once more
// than the copy does) and writes each tile into up to 256 separate runs.  The tile
// form sorts each tile by bucket in place:
//
//   k_tsort      : per tile: rank in shared memory, tq[tile] = the tile's keys in
//                  bucket order (one contiguous, coalesced store), jpos[i] = sorted
//                  position of query i, toff[tidx(b, t)] = start | length << 16 of
//                  bucket b's run in tile t
//   k_lookup_wt  : (capi.cu) CTA (bucket b, group of tiles) walks b's runs of its
//                  tiles; CTAs are numbered bucket-major, so the CTAs resident at a
//                  time share one bucket's slice of the tree as in the global form
//   k_tgather    : per tile: out[i] = tres[tile][jpos[i]], every access coalesced
//
// Every run starts on a 32-B boundary (padded to kRunAlign bytes): a run is walked
// at a different time than its neighbours in the same tile, so a sector shared by
// two runs would be read twice from DRAM and written partially twice (a partial
// sector costs a read-modify-write); the walk writes its padding slots too, so every
// result sector it touches is written whole.  Streaming bytes per u64 query: 8 read
// + 10 written (sort), 8 + 8 (walk I/O), 10 read + 8 written (gather) = 52 B plus
// the padding (~1.5 slots per run), against 60 B for hist + scatter + walk + gather.
constexpr uint32_t kRunAlign = 32;
template <uint32_t KS>
__host__ __device__ constexpr uint32_t run_align_keys() { return kRunAlign / KS; }
// slots per tile region: 4096 keys + at most (A - 1) padding slots per bucket
template <uint32_t KS>
__host__ __device__ constexpr uint32_t tile_stride() { return uint32_t(kBucketTile) + kBuckets * (run_align_keys<KS>() - 1); }
// the stride a batch with nb buckets needs (scratch is sized by it; kernels keep the
// 256-bucket maximum for their shared-memory staging)
template <uint32_t KS>
__host__ __device__ constexpr uint32_t tile_stride_rt(uint32_t nb) { return uint32_t(kBucketTile) + nb * (run_align_keys<KS>() - 1); }
// run table: [group of 8 tiles][bucket < nb][tile in group], u32 start | len << 16
__device__ __forceinline__ uint64_t tidx(uint32_t b, uint64_t t, uint32_t nb) {
    return ((t / kHistGroup) * nb + b) * kHistGroup + (t % kHistGroup);
}
__host__ __device__ constexpr uint64_t tidx_entries(uint64_t tiles, uint32_t nb) {
    return ((tiles + kHistGroup - 1) / kHistGroup) * kHistGroup * nb;
}

// VEC (batch 16-B aligned; the default): keys arrive in 16-B loads, a thread's keys
// are pairs (u64) / quads (u32) of consecutive queries, and their sorted slots leave
// as one 4-B / 8-B jpos store; capped at 64 registers (4 CTAs/SM).  c3: 3.46 -> 3.26
// ms per 2^30 against the strided 8-B-load variant (profiles/r02/tile_form.txt).
template <class Key, bool VEC = false>
__global__ void __launch_bounds__(kBucketThreads, VEC ? 4 : 1) k_tsort(const void* __restrict__ q, uint64_t n, ByteBucket pf,
                                                        uint32_t nb, void* __restrict__ tq,
                                                        uint16_t* __restrict__ jpos, uint32_t* __restrict__ toff) {
    static_assert(Key::kKind == 1 || Key::kKind == 2, "integer keys");
    constexpr uint32_t KS = Key::kKind == 2 ? 8 : 4;
    constexpr uint32_t A = run_align_keys<KS>();
    constexpr uint32_t TS = tile_stride<KS>();
    __shared__ __align__(16) uint8_t skeys[TS * KS];
    __shared__ unsigned int h[kBuckets];
    __shared__ unsigned int loc[kBuckets];
    __shared__ unsigned int wtot[kBucketThreads / 32];
    __shared__ unsigned int ptot;
    h[threadIdx.x] = 0;
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    __syncthreads();
    // item r of this thread is tile position jof(r): strided (plain) or in runs of PER
    constexpr uint32_t PER = VEC ? 16 / KS : 1;
    auto jof = [](int r) -> uint32_t {
        return VEC ? (uint32_t(r / PER) * kBucketThreads + threadIdx.x) * PER + uint32_t(r % PER)
                   : uint32_t(r) * kBucketThreads + threadIdx.x;
    };
    uint64_t kv[kBucketItems];
    if (VEC) {
#pragma unroll
        for (int r = 0; r < kBucketItems; r += PER) {                  // all loads first
            const uint32_t j = jof(r);
            uint4 v = make_uint4(0, 0, 0, 0);
            if (j + PER <= cnt) v = __ldcs((const uint4*)((const uint8_t*)q + (base + j) * KS));
            else
                for (uint32_t e = 0; e < PER; e++)
                    if (j + e < cnt) {                                 // ragged end of the batch
                        if (KS == 8) {
                            const uint64_t x = __ldcs((const unsigned long long*)q + base + j + e);
                            (&v.x)[2 * e] = uint32_t(x);
                            (&v.x)[2 * e + 1] = uint32_t(x >> 32);
                        } else {
                            (&v.x)[e] = __ldcs((const unsigned int*)q + base + j + e);
                        }
                    }
            if (KS == 8) {
                kv[r] = uint64_t(v.x) | (uint64_t(v.y) << 32);
                kv[r + 1] = uint64_t(v.z) | (uint64_t(v.w) << 32);
            } else {
                kv[r] = v.x;
                kv[r + 1] = v.y;
                kv[r + 2] = v.z;
                kv[r + 3] = v.w;
            }
        }
    } else {
#pragma unroll
        for (int r = 0; r < kBucketItems; r++) {                       // all loads first
            const uint32_t j = jof(r);
            kv[r] = 0;
            if (j < cnt)
                kv[r] = Key::kKind == 2 ? uint64_t(__ldcs((const unsigned long long*)q + base + j))
                                        : uint64_t(__ldcs((const unsigned int*)q + base + j));
        }
    }
    uint32_t br[kBucketItems];                                         // bucket << 16 | rank
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t j = jof(r);
        br[r] = 0xFFFFFFFFu;
        if (j < cnt) {
            const uint32_t b = Key::kKind == 2 ? pf.of(KeyU64{kv[r]}) : pf.of(KeyU32{uint32_t(kv[r])});
            br[r] = (b << 16) | atomicAdd(&h[b], 1u);
        }
    }
    __syncthreads();
    const unsigned int c = h[threadIdx.x];
    const unsigned int pc = (c + A - 1) & ~(A - 1);                     // padded run
    const unsigned int lb = block_excl_scan256(pc, wtot);
    loc[threadIdx.x] = lb;
    if (threadIdx.x < nb) toff[tidx(threadIdx.x, blockIdx.x, nb)] = lb | (c << 16);
    if (threadIdx.x == kBucketThreads - 1) ptot = lb + pc;
    __syncthreads();
#pragma unroll
    for (int r0 = 0; r0 < kBucketItems; r0 += PER) {
        uint32_t js[PER];
#pragma unroll
        for (int e = 0; e < int(PER); e++) {
            const int r = r0 + e;
            js[e] = 0;
            if (br[r] != 0xFFFFFFFFu) {
                const uint32_t j = loc[br[r] >> 16] + (br[r] & 0xFFFFu);
                if (Key::kKind == 2) ((uint64_t*)skeys)[j] = kv[r];
                else ((uint32_t*)skeys)[j] = uint32_t(kv[r]);
                js[e] = j;
                if (!VEC) __stcs((unsigned short*)jpos + base + jof(r), (unsigned short)j);
            }
        }
        if (VEC) {
            const uint32_t j = jof(r0);
            if (j + PER <= cnt) {
                if (PER == 2) __stcs((unsigned int*)(jpos + base + j), js[0] | (js[PER > 1 ? 1 : 0] << 16));
                else __stcs((uint2*)(jpos + base + j), make_uint2(js[0] | (js[PER > 1 ? 1 : 0] << 16),
                                                                  js[PER > 2 ? 2 : 0] | (js[PER > 3 ? 3 : 0] << 16)));
            } else {
                for (uint32_t e = 0; e < PER; e++)
                    if (j + e < cnt) jpos[base + j + e] = uint16_t(js[e]);
            }
        }
    }
    __syncthreads();
    // the sorted, padded tile -> tq in 16-B stores (every run and the region are
    // 32-B aligned; padding slots carry stale shared memory, never read as keys)
    const uint32_t nv = ptot * KS / 16;
    const uint32_t ts = tile_stride_rt<KS>(nb);                        // this batch's tile stride
    uint4* dst = (uint4*)((uint8_t*)tq + uint64_t(blockIdx.x) * ts * KS);
#pragma unroll 4
    for (uint32_t v = threadIdx.x; v < nv; v += kBucketThreads) __stcs(dst + v, ((const uint4*)skeys)[v]);
}

// Tile sort of a byte-string batch (32-B slots + lengths).  A key is exactly one
// 32-B sector, so no staging is needed: pass 1 reads each query's length and the
// one key byte its bucket needs and ranks it in shared memory; pass 2 copies the
// whole slot (an L2 hit: pass 1 brought its sector in) to its sorted slot -- a
// full-sector store -- with its length and jpos.  Runs need no padding (A = 1).
static __global__ void __launch_bounds__(kBucketThreads) k_tsort_bytes(const uint8_t* __restrict__ q,
                                                                     const uint8_t* __restrict__ lens, uint64_t n,
                                                                     ByteBucket pf, uint32_t nb, uint8_t* __restrict__ tq,
                                                                     uint8_t* __restrict__ tlen, uint16_t* __restrict__ jpos,
                                                                     uint32_t* __restrict__ toff) {
    constexpr uint32_t TS = tile_stride<32>();
    __shared__ unsigned int h[kBuckets];
    __shared__ unsigned int loc[kBuckets];
    __shared__ unsigned int wtot[kBucketThreads / 32];
    h[threadIdx.x] = 0;
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    __syncthreads();
    uint32_t br[kBucketItems];                                         // bucket << 16 | rank
    const uint32_t d = pf.depth & 0xFFu, sh = pf.depth >> 8;
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        // plain loads (not evict-first): the key's sector must still be in L2 for pass 2
        const uint32_t j = uint32_t(r) * kBucketThreads + threadIdx.x;
        br[r] = 0xFFFFFFFFu;
        if (j < cnt) {
            const uint32_t l = lens[base + j];
            br[r] = d < l ? uint32_t(q[(base + j) * 32 + d]) >> sh : 0u;
        }
    }
#pragma unroll
    for (int r = 0; r < kBucketItems; r++)
        if (br[r] != 0xFFFFFFFFu) br[r] = (br[r] << 16) | atomicAdd(&h[br[r]], 1u);
    __syncthreads();
    const unsigned int c = h[threadIdx.x];
    const unsigned int lb = block_excl_scan256(c, wtot);
    loc[threadIdx.x] = lb;
    if (threadIdx.x < nb) toff[tidx(threadIdx.x, blockIdx.x, nb)] = lb | (c << 16);
    __syncthreads();
    uint8_t* dq = tq + uint64_t(blockIdx.x) * TS * 32;
    uint8_t* dl = tlen + uint64_t(blockIdx.x) * TS;
#pragma unroll 4
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t jt = uint32_t(r) * kBucketThreads + threadIdx.x;
        if (br[r] == 0xFFFFFFFFu) continue;
        const uint32_t j = loc[br[r] >> 16] + (br[r] & 0xFFFFu);
        const uint4* src = (const uint4*)(q + (base + jt) * 32);
        const uint4 a = __ldcs(src), b = __ldcs(src + 1);
        __stcs((uint4*)(dq + uint64_t(j) * 32), a);
        __stcs((uint4*)(dq + uint64_t(j) * 32) + 1, b);
        dl[j] = lens[base + jt];
        __stcs((unsigned short*)jpos + base + jt, (unsigned short)j);
    }
}

// The same with 1024 threads per tile, 4 keys per thread held in registers: every
// slot is read from DRAM once (the two-pass form re-reads the slots whose sector
// left L2 between its passes: 26.7 instead of 17.7 GB per 2^29 c4 queries).
static __global__ void __launch_bounds__(1024) k_tsort_bytes1k(const uint8_t* __restrict__ q,
                                                             const uint8_t* __restrict__ lens, uint64_t n,
                                                             ByteBucket pf, uint32_t nb, uint8_t* __restrict__ tq,
                                                             uint8_t* __restrict__ tlen, uint16_t* __restrict__ jpos,
                                                             uint32_t* __restrict__ toff) {
    constexpr uint32_t TS = tile_stride<32>();
    constexpr int IT = kBucketTile / 1024;
    __shared__ unsigned int h[kBuckets];
    __shared__ unsigned int loc[kBuckets];
    __shared__ unsigned int wtot[kBuckets / 32];
    if (threadIdx.x < kBuckets) h[threadIdx.x] = 0;
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    const uint32_t d = pf.depth & 0xFFu, sh = pf.depth >> 8;
    uint4 ka[IT], kb[IT];
    uint32_t ln[IT];
#pragma unroll
    for (int r = 0; r < IT; r++) {                                     // all loads first
        const uint32_t j = uint32_t(r) * 1024 + threadIdx.x;
        ka[r] = kb[r] = make_uint4(0, 0, 0, 0);
        ln[r] = 0;
        if (j < cnt) {
            const uint4* src = (const uint4*)(q + (base + j) * 32);
            ka[r] = __ldcs(src);
            kb[r] = __ldcs(src + 1);
            ln[r] = __ldcs(lens + base + j);
        }
    }
    __syncthreads();
    uint32_t br[IT];
#pragma unroll
    for (int r = 0; r < IT; r++) {
        const uint32_t j = uint32_t(r) * 1024 + threadIdx.x;
        br[r] = 0xFFFFFFFFu;
        if (j < cnt) {
            const uint4 v = d < 16 ? ka[r] : kb[r];
            const uint32_t wi = (d >> 2) & 3;
            const uint32_t w = wi == 0 ? v.x : wi == 1 ? v.y : wi == 2 ? v.z : v.w;
            const uint32_t b = d < ln[r] ? ((w >> (8 * (d & 3))) & 0xFFu) >> sh : 0u;
            br[r] = (b << 16) | atomicAdd(&h[b], 1u);
        }
    }
    __syncthreads();
    if (threadIdx.x < kBuckets) {                                      // exclusive scan of the 256 counts
        const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
        const uint32_t c = h[threadIdx.x];
        uint32_t x = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= uint32_t(o)) x += y;
        }
        if (lane == 31) wtot[warp] = x;
        __syncwarp();
        h[threadIdx.x] = x - c;                                        // warp-exclusive, fixed up below
    }
    __syncthreads();
    if (threadIdx.x < kBuckets) {
        uint32_t before = 0;
        for (uint32_t w = 0; w < (threadIdx.x >> 5); w++) before += wtot[w];
        loc[threadIdx.x] = h[threadIdx.x] + before;
    }
    __syncthreads();
    if (threadIdx.x < nb) {
        const uint32_t lb = loc[threadIdx.x];
        const uint32_t end = threadIdx.x + 1 < nb ? loc[threadIdx.x + 1] : cnt;
        toff[tidx(threadIdx.x, blockIdx.x, nb)] = lb | ((end - lb) << 16);
    }
    uint8_t* dq = tq + uint64_t(blockIdx.x) * TS * 32;
    uint8_t* dl = tlen + uint64_t(blockIdx.x) * TS;
#pragma unroll
    for (int r = 0; r < IT; r++) {
        const uint32_t jt = uint32_t(r) * 1024 + threadIdx.x;
        if (br[r] == 0xFFFFFFFFu) continue;
        const uint32_t j = loc[br[r] >> 16] + (br[r] & 0xFFFFu);
        __stcs((uint4*)(dq + uint64_t(j) * 32), ka[r]);
        __stcs((uint4*)(dq + uint64_t(j) * 32) + 1, kb[r]);
        dl[j] = uint8_t(ln[r]);
        __stcs((unsigned short*)jpos + base + jt, (unsigned short)j);
    }
}

// Per tile: the tile's padded, sorted results (written by k_lookup_wt) -> shared
// memory in 16-B cp.async copies, then out[i] = sres[jpos[i]] (coalesced).
__device__ __forceinline__ void cp_async16(void* smem, const void* g) {
    const unsigned sa = unsigned(__cvta_generic_to_shared(smem));
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sa), "l"(g));
}
template <uint32_t KS>
__global__ void __launch_bounds__(kBucketThreads) k_tgather(const uint64_t* __restrict__ tres,
                                                          const uint16_t* __restrict__ jpos,
                                                          const uint32_t* __restrict__ toff, uint32_t nb, uint64_t n,
                                                          uint64_t* __restrict__ out) {
    constexpr uint32_t TS = tile_stride<KS>();
    constexpr uint32_t A = run_align_keys<KS>();
    __shared__ __align__(16) uint64_t sres[TS];
    const uint64_t base = uint64_t(blockIdx.x) * kBucketTile;
    const uint32_t cnt = uint32_t(n - base < uint64_t(kBucketTile) ? n - base : kBucketTile);
    uint16_t jp[kBucketItems];
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t k = uint32_t(r) * kBucketThreads + threadIdx.x;
        jp[r] = k < cnt ? __ldcs(jpos + base + k) : 0;
    }
    const uint32_t e = toff[tidx(nb - 1, blockIdx.x, nb)];             // last run: start | len << 16
    const uint32_t ptot = (e & 0xFFFFu) + (((e >> 16) + A - 1) & ~(A - 1));
    const uint64_t* src = tres + uint64_t(blockIdx.x) * tile_stride_rt<KS>(nb);
    const uint32_t nv = (ptot + 1) / 2;                                 // ptot is a multiple of A (even)
#pragma unroll 4
    for (uint32_t v = threadIdx.x; v < nv; v += kBucketThreads) cp_async16(&sres[2 * v], src + 2 * v);
    cp_async_wait_all();
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kBucketItems; r++) {
        const uint32_t k = uint32_t(r) * kBucketThreads + threadIdx.x;
        if (k < cnt) __stcs((unsigned long long*)out + base + k, (unsigned long long)sres[jp[r]]);
    }
}

}  // namespace cuart
