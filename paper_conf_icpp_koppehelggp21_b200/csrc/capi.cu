// capi.cu — the C ABI (include/cuart.h): device index, lookup / update kernels
// for sm_100a, host-buffer pipelines, introspection.
//
// Kernels:
//   k_lookup<Key>  : PAPER.md Fig. 3 lookup within the per-type buffers.
//   k_upd1<Key>    : update stage 1 (§3.4): lookup returning the leaf
//                    location, then register the op index as the leaf's writer
//                    if it is larger than the registered one.
//   k_upd2         : update stage 2: after the grid-wide synchronisation
//                    (the kernel boundary, reading C13), the op whose index is
//                    the registered maximum stores its value.
// Conflict registration (B200 reading of the paper's atomic hash table, P:143,
// ref. [4]): a dense per-leaf 64-bit word winner[leaf] updated with atomicMax of
// (epoch << 32 | op index).  Same semantics as the hash table keyed by leaf
// location storing the maximum op index: the highest op index per leaf wins.
// The epoch in the high half makes every earlier batch's entries smaller, so no
// reset pass is needed between batches (reading C12/§8(a) a9).
#include <cuda_runtime.h>
#include <string.h>

#include <stdlib.h>

#include <atomic>
#include <mutex>
#include <utility>
#include <vector>
#include <new>

#include "../../include/cuart.h"
#include "bucket.cuh"
#include "builder.h"
#include "kernels.cuh"

using namespace cuart;

#include "index.h"

std::atomic<uint64_t> g_cuart_launches{0};   // also counted by route.cu

static void drop_kevents(cuart_index* h) {
    for (auto& e : h->kev) {
        cudaEventDestroy(e.first);
        cudaEventDestroy(e.second);
    }
    h->kev.clear();
    h->klookups = 0;
    h->kslice = 0;
}   // also counted by route.cu

#define CU_TRY(x)                                   \
    do {                                            \
        cudaError_t e_ = (x);                       \
        if (e_ != cudaSuccess) {                    \
            return e_ == cudaErrorMemoryAllocation ? CUART_ERR_OOM : CUART_ERR_CUDA; \
        }                                           \
    } while (0)

// ============================================================================ kernels
// SEG: out is ignored, result i goes to so.at(i) (fused multi-GPU return, §8(e)).
template <class Key, int POL, bool SEG = false, int TPB = 256>
__global__ void __launch_bounds__(TPB, Key::kKind == 3 && TPB == 256 ? 8 : 1) k_lookup(DevIndex ix, const void* __restrict__ q,
                                                const uint8_t* __restrict__ lens, uint64_t n,
                                                uint64_t* __restrict__ out, SegOut so = SegOut{}) {
    const Loader<POL> ld;
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += stride) {
        const Key key = Key::template load<POL != 0>(q, lens, i);
        uint64_t val = kMiss;
        const uint64_t leaf = find_leaf(ix, ld, key, start_link(ix, ld, key), val);
        const uint64_t r = leaf ? val : kMiss;
        uint64_t* dst = SEG ? so.at(i) : out + i;
        if (POL != 0) __stcs((unsigned long long*)dst, (unsigned long long)r);
        else *dst = r;
    }
}

// Pre-bucketed walk from the wide root table with Q queries per thread in lockstep
// phases (integer keys): all Q keys, then all Q wide entries, then all Q leaf
// records are requested before any of them is used, so a thread keeps Q
// independent dependent-load chains in flight (the one-query walk is bound by the
// latency of its chain: 64 warps/SM x 32 queries per ~2 us).  Queries whose path
// is not "wide entry -> leaf" finish with the generic find_leaf.  Results are
// identical to k_lookup.  TPB = 64 by default (a CTA's slot frees when its slowest
// warp ends); LP = leaf-load cache policy: evict_last by default, since in the
// bucketed walk a leaf is re-read by the hit queries of its bucket window (c3:
// 8.91 -> 8.42 ms per 2^30 against the direct walk's evict_first + L2::64B).
// The lockstep walk of Q already-loaded integer keys from the wide root table
// (shared by k_lookup_wq and the tile-form walk k_lookup_wt).
template <class Key, int POL, int Q, int LP>
__device__ __forceinline__ void wq_walk(const DevIndex& ix, const Loader<POL>& ld, const Key (&k)[Q], uint64_t (&res)[Q]) {
    U8x32 e[Q];
#pragma unroll
    for (int j = 0; j < Q; j++) e[j] = ld.lutv8(ix.lutw + k[j].prefix(ix.lut_bytes) * 4);
    uint64_t link[Q];
#pragma unroll
    for (int j = 0; j < Q; j++) link[j] = decode_wide(ix, ld, k[j], e[j]);
    // one inline N4 step (the wide entry's node had an inner child: on c3 a depth-4
    // N4), so only deeper paths take the generic find_leaf loop
#pragma unroll
    for (int j = 0; j < Q; j++)
        if (link_type(link[j]) == T_N4) e[j] = ld.nodev8(ix.base[T_N4] + link_index(link[j]) * record_bytes(T_N4));
#pragma unroll
    for (int j = 0; j < Q; j++) {
        if (link_type(link[j]) != T_N4) continue;
        const uint32_t aux = link_aux(link[j]);
        const int c = aux < k[j].len() ? find_key4(e[j].w[0], k[j].byte(aux)) : -1;
        if (c < 0) link[j] = 0;
        else if (c == 3) link[j] = ld.node64(ix.base[T_N4] + link_index(link[j]) * record_bytes(T_N4) + kN4Child + 24);
        else {
            const uint32_t lo = c == 0 ? e[j].w[2] : c == 1 ? e[j].w[4] : e[j].w[6];
            const uint32_t hi = c == 0 ? e[j].w[3] : c == 1 ? e[j].w[5] : e[j].w[7];
            link[j] = uint64_t(lo) | (uint64_t(hi) << 32);
        }
    }
    uint4 r[Q];
#pragma unroll
    for (int j = 0; j < Q; j++)
        if (link_type(link[j]) == T_LEAF8) r[j] = ld.template leafv4_b<LP>(ix.base[T_LEAF8] + link_index(link[j]) * record_bytes(T_LEAF8));
#pragma unroll
    for (int j = 0; j < Q; j++) {
        res[j] = kMiss;
        if (link_type(link[j]) == T_LEAF8) {
            const uint64_t kb = Key::kKind == 2 ? bswap64(uint64_t(k[j].k)) : uint64_t(__byte_perm(uint32_t(k[j].k), 0, 0x0123));
            if (link_aux(link[j]) == k[j].len() && (uint64_t(r[j].x) | (uint64_t(r[j].y) << 32)) == kb)
                res[j] = uint64_t(r[j].z) | (uint64_t(r[j].w) << 32);
        } else if (link[j]) {
            uint64_t val = kMiss;
            if (find_leaf(ix, ld, k[j], link[j], val)) res[j] = val;
        }
    }
}

template <class Key, int POL, int Q, int TPB = 256, bool SEG = false, int LP = 3>
__global__ void __launch_bounds__(TPB) k_lookup_wq(DevIndex ix, const void* __restrict__ q,
                                                   const uint8_t* __restrict__ lens, uint64_t n,
                                                   uint64_t* __restrict__ out, SegOut so = SegOut{}) {
    static_assert(Key::kKind == 1 || Key::kKind == 2, "integer keys");
    const Loader<POL> ld;
    const uint64_t i0 = uint64_t(blockIdx.x) * (TPB * Q) + threadIdx.x;
    Key k[Q];
#pragma unroll
    for (int j = 0; j < Q; j++) {
        const uint64_t i = i0 + uint64_t(j) * TPB;
        k[j] = i < n ? Key::template load<true>(q, lens, i) : Key{0};
    }
    uint64_t res[Q];
    wq_walk<Key, POL, Q, LP>(ix, ld, k, res);
#pragma unroll
    for (int j = 0; j < Q; j++) {
        const uint64_t i = i0 + uint64_t(j) * TPB;
        if (i >= n) continue;
        uint64_t* dst = SEG ? so.at(i) : out + i;
        __stcs((unsigned long long*)dst, (unsigned long long)res[j]);
    }
}

// Tile-form K-BUCKET walk (bucket.cuh k_tsort): CTA (b, g) walks bucket b's runs of
// the tg tiles of group g -- the padded runs are concatenated in tile order, thread p
// of a round takes position p of the concatenation (a binary search over the run
// prefix in shared memory gives its tile), and the result goes to the same
// tile-sorted position, which k_tgather returns to query order; a padding position
// writes CUART_MISS so that every result sector is written whole.  CTAs are numbered
// bucket-major, so the CTAs resident at a time walk one bucket's slice of the tree
// (the locality of the global bucketed order) without a global scatter.  WIDE: the
// lockstep wide-table walk of k_lookup_wq; else the generic walk from the LINKS root
// table.  No barrier inside the round loop: each warp runs its rounds independently.
template <class Key, int Q, int TPB, int LP, bool WIDE, int MINB = 1>
__global__ void __launch_bounds__(TPB, MINB) k_lookup_wt(DevIndex ix, const void* __restrict__ tq,
                                                         const uint32_t* __restrict__ toff, uint64_t n, uint32_t nb,
                                                         uint32_t tg, uint32_t ngroups, uint64_t* __restrict__ tres,
                                                         const uint8_t* __restrict__ tlen = nullptr) {
    static_assert(Key::kKind == 1 || Key::kKind == 2 || (Key::kKind == 3 && !WIDE), "integer keys or byte strings");
    constexpr uint32_t KS = Key::kKind == 2 ? 8 : Key::kKind == 1 ? 4 : 32;
    constexpr uint32_t A = run_align_keys<KS>();
    constexpr uint32_t TS = tile_stride<KS>();
    // up to kTgMax tiles per CTA; the first two warps scan their run lengths
    constexpr uint32_t kTgMax = 64;
    static_assert(TPB >= kTgMax, "two warps build the run table");
    __shared__ uint32_t pre[kTgMax + 1];               // run start in the concatenation; pre[tg..]: sentinel
    __shared__ uint2 de[kTgMax];                       // {slot - position, end of the live part of the run}
    __shared__ uint32_t wtot[2];
    __shared__ uint32_t total;
    const uint32_t b = blockIdx.x / ngroups, g = blockIdx.x - b * ngroups;
    const uint64_t tiles = (n + kBucketTile - 1) / kBucketTile;
    const uint32_t ts = tile_stride_rt<KS>(nb);       // tile stride of this batch (<= TS)
    const uint64_t gbase = uint64_t(g) * tg * ts;      // first slot of the group (tg * ts < 2^19)
    const uint32_t i = threadIdx.x;
    const bool valid = i < tg && uint64_t(g) * tg + i < tiles;
    if (i < kTgMax) {
        const uint32_t lane = i & 31;
        const uint32_t e = valid ? toff[tidx(b, uint64_t(g) * tg + i, nb)] : 0u;
        const uint32_t len = e >> 16, plen = (len + A - 1) & ~(A - 1);
        uint32_t x = plen;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, d);
            if (lane >= uint32_t(d)) x += y;
        }
        if (lane == 31) wtot[i >> 5] = x;
        pre[i] = x - plen;                             // exclusive within the warp (fixed up below)
        de[i] = make_uint2(i * ts + (e & 0xFFFFu), len);
    }
    __syncthreads();
    if (i < kTgMax) {
        const uint32_t p_run = pre[i] + (i >= 32 ? wtot[0] : 0u);
        const uint2 r = de[i];
        pre[i] = valid ? p_run : 0xFFFFFFFFu;           // invalid lanes are never selected
        de[i] = make_uint2(r.x - p_run, p_run + r.y);
        if (i == 0) {
            total = wtot[0] + wtot[1];
            pre[kTgMax] = 0xFFFFFFFFu;
        }
    }
    __syncthreads();
    const uint32_t T = total;
    uint32_t lo = 0;                                   // tile of the thread's last position (only moves forward)
    const uint8_t* kq = (const uint8_t*)tq + gbase * KS;
    const uint8_t* kl = Key::kKind == 3 ? tlen + gbase : nullptr;
    unsigned long long* rq = (unsigned long long*)tres + gbase;
    constexpr uint32_t kDead = 0x80000000u;            // padding slot: no walk, CUART_MISS written
#pragma unroll 1
    for (uint32_t p0 = 0; p0 < T; p0 += TPB * Q) {
        uint32_t rel[Q];                               // slot relative to gbase | kDead, or ~0 (past the end)
        Key k[Q];
#pragma unroll
        for (int j = 0; j < Q; j++) {
            const uint32_t p = p0 + uint32_t(j) * TPB + threadIdx.x;
            // largest tile whose run starts at or before p: positions grow by TPB per
            // step and runs average 4096 / nb slots, so this is 0-2 steps forward
#pragma unroll 1
            while (pre[lo + 1] <= p) lo++;
            const uint2 d = de[lo];
            rel[j] = p >= T ? ~0u : (p + d.x) | (p < d.y ? 0u : kDead);
            if (rel[j] < kDead) k[j] = Key::template load<true>(kq, kl, rel[j]);
            else k[j] = Key{};
        }
        const Loader<5> ld;                            // per round: the policies are not held across rounds
        uint64_t res[Q];
        if constexpr (WIDE) {
            wq_walk<Key, 5, Q, LP>(ix, ld, k, res);
        } else {
#pragma unroll
            for (int j = 0; j < Q; j++) {
                uint64_t val = kMiss;
                res[j] = rel[j] < kDead && find_leaf(ix, ld, k[j], start_link(ix, ld, k[j]), val) ? val : kMiss;
            }
        }
#pragma unroll
        for (int j = 0; j < Q; j++)
            if (rel[j] != ~0u) __stcs(rq + (rel[j] & ~kDead), (unsigned long long)(rel[j] < kDead ? res[j] : kMiss));
    }
}

// f4 (P:126 option 2): the walk for CUART_KEY_LONG queries.  A query ending at a
// host-leaf link returns the leaf's host index with sig[i] = 1 ("the CPU needs to
// compare the complete key"); every other query is final (sig[i] = 0).
template <int POL>
__global__ void __launch_bounds__(256) k_lookup_long(DevIndex ix, const uint8_t* __restrict__ q,
                                                     const uint64_t* __restrict__ off, uint64_t n,
                                                     uint64_t* __restrict__ out, uint8_t* __restrict__ sig) {
    const Loader<POL> ld;
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += stride) {
        const KeyLong key = KeyLong::load<true>(q, (const uint8_t*)off, i);
        uint64_t val = kMiss;
        const uint64_t leaf = find_leaf(ix, ld, key, start_link(ix, ld, key), val);
        const bool host = leaf && link_type(leaf) == T_LEAF_HOST;
        out[i] = host ? link_index(leaf) : (leaf ? val : kMiss);
        sig[i] = host ? 1 : 0;
    }
}

// a5 + a4 together: the pre-bucketed walk with the bucket's slice of the RANK root
// table in shared memory.  Persistent CTAs visit the buckets in order; for
// bucket b every CTA walks an equal contiguous share of b's run of the bucketed
// batch, so at any moment all SMs work inside one bucket (its tree slice stays
// L2-resident, exactly as when k_lookup walks the bucketed batch) while the table
// entries of prefix C.b.* (C = the root's compressed prefix, d bytes) are read from
// shared memory instead of L2: one L2 request less per query.  A query whose
// prefix is not C.b (an absent key) reads the global table.  The slice refill is
// S bytes per CTA per bucket (S = 2^shift entries, 64 KiB for k = 3, d = 0).
constexpr int kSliceThreads = 1024;
template <class Key, int POL>
__global__ void __launch_bounds__(kSliceThreads, 2) k_lookup_slice(DevIndex ix, const void* __restrict__ q, uint64_t n,
                                                                   uint64_t* __restrict__ out,
                                                                   const unsigned int* __restrict__ bases, uint64_t e0,
                                                                   uint32_t shift) {
    extern __shared__ uint4 slut[];
    const Loader<POL> ld;
    const uint64_t S = uint64_t(1) << shift;
    const uint32_t nv4 = uint32_t(S >> 4);                    // 1 B per entry, in 16-B units
    for (uint32_t b = 0; b < uint32_t(kBuckets); b++) {
        const uint64_t lo = bases[b], hi = b + 1 < uint32_t(kBuckets) ? uint64_t(bases[b + 1]) : n;
        if (lo >= hi) continue;
        const uint64_t per = (hi - lo + gridDim.x - 1) / gridDim.x;
        const uint64_t s0 = lo + per * blockIdx.x;
        const uint64_t s1 = s0 + per < hi ? s0 + per : hi;
        if (s0 >= s1) continue;                                // uniform over the CTA
        const uint64_t E0 = e0 | (uint64_t(b) << shift);
        __syncthreads();                                       // the previous slice is no longer read
        const uint4* src = ix.lutr + (E0 >> 5) * 2;
        for (uint32_t k = threadIdx.x; k < nv4; k += blockDim.x)
            slut[k] = POL ? Loader<POL>::v4(src + k, ld.keep) : ld_nc_v4(src + k);
        __syncthreads();
        for (uint64_t i = s0 + threadIdx.x; i < s1; i += blockDim.x) {
            const Key key = Key::template load<true>(q, nullptr, i);
            const uint64_t p = key.prefix(ix.lut_bytes);
            uint64_t link;
            if (p - E0 < S) {
                const uint4* sp = slut + ((p - E0) >> 5) * 2;
                const uint4 a = sp[0], c = sp[1];
                U8x32 blk;
                blk.w[0] = a.x; blk.w[1] = a.y; blk.w[2] = a.z; blk.w[3] = a.w;
                blk.w[4] = c.x; blk.w[5] = c.y; blk.w[6] = c.z; blk.w[7] = c.w;
                link = decode_lut_rank(ix, ld, blk, p);
            } else {
                link = start_link(ix, ld, key);
            }
            uint64_t val = kMiss;
            const uint64_t leaf = find_leaf(ix, ld, key, link, val);
            __stcs((unsigned long long*)out + i, (unsigned long long)(leaf ? val : kMiss));
        }
    }
}

__device__ __forceinline__ uint64_t global_leaf_id(const DevIndex& ix, uint64_t leaf) {
    const uint32_t t = link_type(leaf);
    return (t == T_LEAF8 ? ix.leaf_base[5] : t == T_LEAF16 ? ix.leaf_base[6] : ix.leaf_base[7]) + link_index(leaf);
}

// Stage 1 of the two-stage update (Fig. 6).  DEL: the batch may carry
// deletes ("the same implementation ... signaling a deletion through a
// nil pointer"): is_delete[i] != 0 (or is_delete == NULL: every op deletes); the
// parent's child slot of the located leaf is recorded for stage 2 to unlink.
// A located leaf holding the tombstone (value == CUART_MISS) was deleted earlier
// and counts as absent (reading C17/C18).
__device__ __forceinline__ uint64_t* winner_word(const DevIndex& ix, uint64_t leaf) {
#if CUART_COLOCATED_WINNER
    const uint32_t t = link_type(leaf);
    return (uint64_t*)(ix.base[t] + link_index(leaf) * record_bytes(t) + leaf_winner_off(t));
#else
    return &ix.winner[global_leaf_id(ix, leaf)];
#endif
}

// Epoch wrap (every 2^32 - 2 update batches): zero every conflict word.
__global__ void k_clear_winners(DevIndex ix, uint64_t n8, uint64_t n16, uint64_t n32) {
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n8 + n16 + n32; i += stride) {
        const uint32_t t = i < n8 ? T_LEAF8 : i < n8 + n16 ? T_LEAF16 : T_LEAF32;
        const uint64_t idx = i < n8 ? i : i < n8 + n16 ? i - n8 : i - n8 - n16;
        *winner_word(ix, make_link(t, 0, idx)) = 0;
    }
}

template <class Key, int POL, bool DEL>
__global__ void __launch_bounds__(256) k_upd1(DevIndex ix, const void* __restrict__ q, const uint8_t* __restrict__ lens,
                                              const uint64_t* __restrict__ vals, const uint8_t* __restrict__ is_delete,
                                              uint64_t n, uint64_t epoch_hi, uint64_t* __restrict__ leafref,
                                              uint64_t* __restrict__ slotref, const uint32_t* __restrict__ opidx) {
    const Loader<POL> ld;
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += stride) {
        const Key key = Key::template load<POL != 0>(q, lens, i);
        const bool del = DEL && (is_delete == nullptr || is_delete[i]);
        uint64_t val, slot = 0;
        uint64_t leaf = find_leaf<Key, POL, DEL>(ix, ld, key, start_link<Key, POL, DEL>(ix, ld, key, &slot), val, &slot);
        if (leaf && val == kMiss) leaf = 0;            // tombstone: deleted by an earlier batch
        if (!del && vals[i] == kMiss) {                // reserved value: op rejected, sticky error
            atomicOr(ix.err, 1u);
            leaf = 0;
        }
        leafref[i] = leaf;
        if (DEL) slotref[i] = slot;
        const uint64_t prio = opidx ? uint64_t(opidx[i]) : i;      // priority = original op index
        // f4: a host leaf (link type 8) is resolved by the host after the kernels
        if (leaf && (Key::kKind != 4 || link_type(leaf) != T_LEAF_HOST))
            atomicMax((unsigned long long*)winner_word(ix, leaf), (unsigned long long)(epoch_hi | prio));
    }
}

// Stage 1 of a pre-bucketed plain update batch (integer keys, wide root table):
// k_upd1's work with Q ops per thread in lockstep phases, as k_lookup_wq (keys,
// values and op indices, then the wide entries, then the leaf records are all
// requested before use).  Same outputs as k_upd1<Key, 5, false>.
template <class Key, int Q, int TPB = 64>
__global__ void __launch_bounds__(TPB) k_upd1_wq(DevIndex ix, const void* __restrict__ q, const uint64_t* __restrict__ vals,
                                                 uint64_t n, uint64_t epoch_hi, uint64_t* __restrict__ leafref,
                                                 const uint32_t* __restrict__ opidx) {
    static_assert(Key::kKind == 1 || Key::kKind == 2, "integer keys");
    const Loader<5> ld;
    const uint64_t i0 = uint64_t(blockIdx.x) * (TPB * Q) + threadIdx.x;
    Key k[Q];
    uint64_t v[Q];
    uint32_t pr[Q];
#pragma unroll
    for (int j = 0; j < Q; j++) {
        const uint64_t i = i0 + uint64_t(j) * TPB;
        const bool ok = i < n;
        k[j] = ok ? Key::template load<true>(q, nullptr, i) : Key{0};
        v[j] = ok ? uint64_t(__ldcs((const unsigned long long*)vals + i)) : 0;
        pr[j] = ok ? (opidx ? __ldcs(opidx + i) : uint32_t(i)) : 0u;
    }
    U8x32 e[Q];
#pragma unroll
    for (int j = 0; j < Q; j++) e[j] = ld.lutv8(ix.lutw + k[j].prefix(ix.lut_bytes) * 4);
    uint64_t link[Q];
#pragma unroll
    for (int j = 0; j < Q; j++) link[j] = decode_wide(ix, ld, k[j], e[j]);
    uint4 r[Q];
#pragma unroll
    for (int j = 0; j < Q; j++)
        if (link_type(link[j]) == T_LEAF8) r[j] = ld.template leafv4_b<3>(ix.base[T_LEAF8] + link_index(link[j]) * record_bytes(T_LEAF8));
#pragma unroll
    for (int j = 0; j < Q; j++) {
        const uint64_t i = i0 + uint64_t(j) * TPB;
        if (i >= n) continue;
        uint64_t leaf = 0, val = kMiss;
        if (link_type(link[j]) == T_LEAF8) {
            const uint64_t kb = Key::kKind == 2 ? bswap64(uint64_t(k[j].k)) : uint64_t(__byte_perm(uint32_t(k[j].k), 0, 0x0123));
            if (link_aux(link[j]) == k[j].len() && (uint64_t(r[j].x) | (uint64_t(r[j].y) << 32)) == kb) {
                leaf = link[j];
                val = uint64_t(r[j].z) | (uint64_t(r[j].w) << 32);
            }
        } else if (link[j]) {
            leaf = find_leaf(ix, ld, k[j], link[j], val);
        }
        if (leaf && val == kMiss) leaf = 0;            // tombstone: deleted by an earlier batch
        if (v[j] == kMiss) {                           // reserved value: op rejected, sticky error
            atomicOr(ix.err, 1u);
            leaf = 0;
        }
        leafref[i] = leaf;
        if (leaf) atomicMax((unsigned long long*)winner_word(ix, leaf), (unsigned long long)(epoch_hi | pr[j]));
    }
}

// Stage 2: after the grid-wide synchronisation (kernel boundary), the op whose
// index is the registered maximum applies: one aligned 8-byte value store,
// or, for a delete, unlink the leaf from its parent slot, clear it (value :=
// tombstone CUART_MISS; key bytes kept so the leaf buffer stays sorted)
// and push its id on the free-leaf list.
template <bool DEL, int TPB = 256>
__global__ void __launch_bounds__(TPB) k_upd2(DevIndex ix, const uint64_t* __restrict__ vals,
                                              const uint8_t* __restrict__ is_delete, uint64_t n, uint64_t epoch_hi,
                                              const uint64_t* __restrict__ leafref, const uint64_t* __restrict__ slotref,
                                              const uint32_t* __restrict__ opidx) {
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += stride) {
        const uint64_t leaf = leafref[i];
        if (!leaf || link_type(leaf) == T_LEAF_HOST) continue;   // f4: host leaves are applied by the host
        const uint64_t gid = global_leaf_id(ix, leaf);
        const uint64_t prio = opidx ? uint64_t(opidx[i]) : i;
        if (__ldcg(winner_word(ix, leaf)) != (epoch_hi | prio)) continue;
        const uint32_t t = link_type(leaf);
        uint64_t* dst = (uint64_t*)(ix.base[t] + link_index(leaf) * record_bytes(t) + leaf_value_off(t));
        if (DEL && (is_delete == nullptr || is_delete[i])) {
            const uint64_t sl = slotref[i];
            if (sl & 1) *(uint32_t*)(sl & ~uint64_t(1)) = 0;       // compact 32-bit LUT entry
            else if (sl) *(uint64_t*)sl = 0;                       // 64-bit link: node child / LUT entry
            if (ix.lutw && sl >= uint64_t(ix.lut) && sl < uint64_t(ix.lut + ix.lut_entries))
                ix.lutw[(sl - uint64_t(ix.lut)) / 8 * 4] = 0;      // the wide table's copy of that entry
            *dst = kMiss;
            const unsigned long long pos = atomicAdd(ix.free_count, 1ull);
            ix.free_list[pos] = uint32_t(gid);
        } else {
            *dst = vals[i];
        }
    }
}

// ============================================================================ helpers
static int grid_for(const cuart_index* h, uint64_t n) {
    uint64_t blocks = (n + 255) / 256;
    // Default: one op per thread (measured fastest on c3: CTAs retire and refill
    // per SM instead of long grid-stride loops).  Tuning knob: a persistent grid.
    uint64_t cap = (uint64_t(1) << 31) - 1;
    if (h->grid_ctas_per_sm > 0) cap = uint64_t(h->num_sms) * h->grid_ctas_per_sm;
    if (blocks > cap) blocks = cap;
    return int(blocks < 1 ? 1 : blocks);
}

static cuart_status check_keys(const cuart_index* h, const cuart_keys* k, size_t n) {
    if (!h || !k) return CUART_ERR_INVALID_ARGUMENT;
    if (k->kind == CUART_KEY_LONG || h->key_kind == CUART_KEY_LONG) return CUART_ERR_INVALID_ARGUMENT;   // *_long calls
    if (n > 0 && k->data == nullptr) return CUART_ERR_INVALID_ARGUMENT;
    if (uint32_t(k->kind) != h->key_kind) return CUART_ERR_INVALID_ARGUMENT;
    if (k->kind == CUART_KEY_BYTES && n > 0 && k->lengths == nullptr) return CUART_ERR_INVALID_ARGUMENT;
    return CUART_OK;
}


static void ktimer_begin(const cuart_index* h, cudaStream_t s, cudaEvent_t& ev0, cudaEvent_t& ev1) {
    ev0 = ev1 = nullptr;
    if (!h->ktimer) return;
    cudaEventCreate(&ev0);
    cudaEventCreate(&ev1);
    cudaEventRecord(ev0, s);
}
static void ktimer_end(const cuart_index* h, cudaStream_t s, cudaEvent_t ev0, cudaEvent_t ev1, uint64_t n,
                       bool slice = false) {
    if (!h->ktimer) return;
    cudaEventRecord(ev1, s);
    cuart_index* hm = const_cast<cuart_index*>(h);
    std::lock_guard<std::mutex> g(hm->kmu);
    hm->kev.push_back({ev0, ev1});
    hm->klookups += n;
    hm->kslice += slice ? 1 : 0;
}

template <class Key>
static cuart_status launch_lookup_slice(const cuart_index* h, const void* bq, uint64_t n, uint64_t* res,
                                        const unsigned int* bases, cudaStream_t s) {
    cudaEvent_t ev0, ev1;
    ktimer_begin(h, s, ev0, ev1);
    const size_t smem = size_t(1) << h->slice_shift;
    k_lookup_slice<Key, 5><<<h->slice_grid, kSliceThreads, smem, s>>>(h->dix, bq, n, res, bases, h->slice_e0,
                                                                     h->slice_shift);
    g_cuart_launches++;
    ktimer_end(h, s, ev0, ev1, n, true);
    CU_TRY(cudaGetLastError());
    return CUART_OK;
}

// a5 pre-bucketing: bucket -> lookup in bucketed order -> gather (bucket.cuh).
// Scratch is stream-ordered (cudaMallocAsync from the device pool, whose release
// threshold is raised at upload so the memory stays mapped between calls), so
// concurrent lookups on several streams stay independent.
template <class Key>
static cuart_status launch_bucketed(const cuart_index* h, const void* q, const uint8_t* lens, uint64_t n, uint64_t* out,
                                    cudaStream_t s, const SegOut* so = nullptr) {
    const size_t ks = Key::kKind == 2 ? 8 : Key::kKind == 1 ? 4 : 32;
    auto al = [](size_t x) { return (x + 255) & ~size_t(255); };
    const uint64_t tiles = (n + kBucketTile - 1) / kBucketTile;
    const size_t o_hist = 0, o_tot = al(hist_entries(tiles) * 4), o_q = o_tot + 2048, o_len = o_q + al(n * ks),
                 o_pos = o_len + al(Key::kKind == 3 ? n : 0), o_res = o_pos + al(n * 2), total = o_res + al(n * 8);
    uint8_t* scr = nullptr;
    cuart_status rc = scratch_alloc(h, (void**)&scr, total, s);
    if (rc != CUART_OK) return rc;
    unsigned int* hist = (unsigned int*)(scr + o_hist);
    unsigned int* tot = (unsigned int*)(scr + o_tot);
    const uint32_t depth = (link_type(h->root) >= T_N4 && link_type(h->root) <= T_N256 ? link_aux(h->root) : 0u) |
                           (h->bucket_shift << 8);
    if ((uintptr_t(q) & 15) == 0) k_bhist<Key, true><<<unsigned(tiles), kBucketThreads, 0, s>>>(q, lens, n, ByteBucket(depth), hist);
    else k_bhist<Key, false><<<unsigned(tiles), kBucketThreads, 0, s>>>(q, lens, n, ByteBucket(depth), hist);
    k_bscan_rows<<<kBuckets >> h->bucket_shift, kBucketThreads, 0, s>>>(hist, tiles, tot);   // rows in use only
    k_bscan<<<1, kBuckets, 0, s>>>(tot, kBuckets >> h->bucket_shift);
    k_bscatter<Key><<<unsigned(tiles), kBucketThreads, bscatter_smem<Key>(), s>>>(
        q, lens, n, ByteBucket(depth), hist, tot, scr + o_q, Key::kKind == 3 ? scr + o_len : nullptr, (uint16_t*)(scr + o_pos));
    g_cuart_launches += 4;
    if (cudaGetLastError() != cudaSuccess) {
        scratch_free(h, scr, s);
        return CUART_ERR_CUDA;
    }
    const uint64_t slice_bytes = uint64_t(1) << h->slice_shift;
    // AUTO = off: measured slower than k_lookup over the bucketed batch on c3 (19.2 vs
    // 15.0 ms per 2^30: the 64-KiB slices take L1 capacity, L2 hit rate 64% -> 49%)
    // and on c2 (3.10 vs 2.57 ms per 2^28: the per-bucket CTA barriers).  Kept as an
    // explicit option (CUART_SLICE_ON) with its parity tests.
    (void)slice_bytes;
    const bool slice = Key::kKind != 3 && h->slice_ok && h->policy == 5 && h->slice_lut == CUART_SLICE_ON &&
                       h->bucket_shift == 0;
    if (slice) rc = launch_lookup_slice<Key>(h, scr + o_q, n, (uint64_t*)(scr + o_res), tot, s);
    else rc = launch_lookup_direct(h, Key::kKind, scr + o_q, Key::kKind == 3 ? scr + o_len : nullptr, n,
                                   (uint64_t*)(scr + o_res), s, nullptr, true);
    if (rc != CUART_OK) {
        scratch_free(h, scr, s);
        return rc;
    }
    if (so) k_bgather<true><<<unsigned(tiles), kBucketThreads, 0, s>>>((const uint64_t*)(scr + o_res),
                                                                        (const uint16_t*)(scr + o_pos), n, hist, tot,
                                                                        nullptr, *so);
    else k_bgather<false><<<unsigned(tiles), kBucketThreads, 0, s>>>((const uint64_t*)(scr + o_res),
                                                                      (const uint16_t*)(scr + o_pos), n, hist, tot, out);
    g_cuart_launches++;
    rc = cudaGetLastError() == cudaSuccess ? CUART_OK : CUART_ERR_CUDA;
    scratch_free(h, scr, s);
    return rc;
}

// a5 pre-bucketing, tile form (bucket.cuh k_tsort / k_tgather, capi.cu k_lookup_wt):
// sort every tile by bucket in place -> walk bucket-major over the tiles' runs ->
// per-tile gather.  Integer keys, results to `out` (no fused multi-GPU return).
template <class Key>
static cuart_status launch_tiled(const cuart_index* h, const void* q, const uint8_t* lens, uint64_t n, uint64_t* out,
                                 cudaStream_t s) {
    constexpr uint32_t KS = Key::kKind == 2 ? 8 : Key::kKind == 1 ? 4 : 32;
    auto al = [](size_t x) { return (x + 255) & ~size_t(255); };
    const uint64_t tiles = (n + kBucketTile - 1) / kBucketTile;
    const uint32_t nb = kBuckets >> h->bucket_shift;
    const uint64_t TS = tile_stride_rt<KS>(nb);       // c3 (64 buckets): 4288 slots per 4096-query tile
    const size_t o_off = 0, o_q = al(tidx_entries(tiles, nb) * 4), o_len = o_q + al(tiles * TS * KS),
                 o_pos = o_len + al(Key::kKind == 3 ? tiles * TS : 0), o_res = o_pos + al(n * 2),
                 total = o_res + al(tiles * TS * 8);
    uint8_t* scr = nullptr;
    cuart_status rc = scratch_alloc(h, (void**)&scr, total, s);
    if (rc != CUART_OK) return rc;
    uint32_t* toff = (uint32_t*)(scr + o_off);
    const uint32_t depth = (link_type(h->root) >= T_N4 && link_type(h->root) <= T_N256 ? link_aux(h->root) : 0u) |
                           (h->bucket_shift << 8);
    if constexpr (Key::kKind == 3) {
        if (h->tsort_b1k)
            k_tsort_bytes1k<<<unsigned(tiles), 1024, 0, s>>>((const uint8_t*)q, lens, n, ByteBucket(depth), nb,
                                                             scr + o_q, scr + o_len, (uint16_t*)(scr + o_pos), toff);
        else
            k_tsort_bytes<<<unsigned(tiles), kBucketThreads, 0, s>>>((const uint8_t*)q, lens, n, ByteBucket(depth), nb,
                                                                    scr + o_q, scr + o_len, (uint16_t*)(scr + o_pos), toff);
    }
    else if (h->tsort_vec && (uintptr_t(q) & 15) == 0)
        k_tsort<Key, true><<<unsigned(tiles), kBucketThreads, 0, s>>>(q, n, ByteBucket(depth), nb, scr + o_q,
                                                                     (uint16_t*)(scr + o_pos), toff);
    else
        k_tsort<Key><<<unsigned(tiles), kBucketThreads, 0, s>>>(q, n, ByteBucket(depth), nb, scr + o_q,
                                                               (uint16_t*)(scr + o_pos), toff);
    g_cuart_launches++;
    if (cudaGetLastError() != cudaSuccess) {
        scratch_free(h, scr, s);
        return CUART_ERR_CUDA;
    }
    // tiles per walk CTA: bucket runs average 4096 / nb keys; ~2048 queries per CTA
    // (16 rounds of 64 threads x 2 queries), at most 32 (one warp builds the prefix).
    // c3 walk per 2^30: 12.3 / 10.8 / 9.7 / 9.4 ms at 4 / 8 / 16 / 32 tiles (the
    // table prologue is paid per CTA)
    uint32_t tg = uint32_t((2048 * uint64_t(nb)) / kBucketTile);
    tg = tg < 1 ? 1 : tg > 64 ? 64 : tg;
    if (h->tile_group) tg = h->tile_group;
    const uint32_t ngroups = uint32_t((tiles + tg - 1) / tg);
    const DevIndex& dx = h->dix_links;
    const bool wide = Key::kKind != 3 && dx.walk_wide && h->policy == 5 && h->ilp > 1;
    cudaEvent_t ev0, ev1;
    ktimer_begin(h, s, ev0, ev1);
    const unsigned g = nb * ngroups;
    uint64_t* tres = (uint64_t*)(scr + o_res);
    // 20 CTAs/SM (48 registers instead of 52, no spill): c3 walk 9.42 -> 9.07 ms per 2^30
    // (profiles/r02/tile_form.txt); 24 CTAs/SM spills (40 registers + 24 B stack)
    if constexpr (Key::kKind == 3) {
        // byte strings: 256-thread CTAs at 8 CTAs/SM (32 registers): c4 walk 32.97 ms per
        // 2^29 against 38.39 (64 threads, 46 registers) and 35.58 (64 threads, 24 CTAs/SM)
        // (profiles/r02/tile_form.txt)
        if (h->wt_tpb == 64) k_lookup_wt<Key, 1, 64, 3, false, 24><<<g, 64, 0, s>>>(dx, scr + o_q, toff, n, nb, tg, ngroups, tres, scr + o_len);
        else if (h->wt_tpb == 128) k_lookup_wt<Key, 1, 128, 3, false, 12><<<g, 128, 0, s>>>(dx, scr + o_q, toff, n, nb, tg, ngroups, tres, scr + o_len);
        else if (h->wt_minb == 6) k_lookup_wt<Key, 1, 256, 3, false, 6><<<g, 256, 0, s>>>(dx, scr + o_q, toff, n, nb, tg, ngroups, tres, scr + o_len);
        else k_lookup_wt<Key, 1, 256, 3, false, 8><<<g, 256, 0, s>>>(dx, scr + o_q, toff, n, nb, tg, ngroups, tres, scr + o_len);
    } else {
        if (wide && h->wt_tpb == 128) k_lookup_wt<Key, 2, 128, 3, true, 10><<<g, 128, 0, s>>>(dx, scr + o_q, toff, n, nb, tg, ngroups, tres);
        else if (wide && h->wt_tpb == 256) k_lookup_wt<Key, 2, 256, 3, true, 5><<<g, 256, 0, s>>>(dx, scr + o_q, toff, n, nb, tg, ngroups, tres);
        else if (wide && h->wt_minb == 1) k_lookup_wt<Key, 2, 64, 3, true, 1><<<g, 64, 0, s>>>(dx, scr + o_q, toff, n, nb, tg, ngroups, tres);
        else if (wide && h->wt_minb == 24) k_lookup_wt<Key, 2, 64, 3, true, 24><<<g, 64, 0, s>>>(dx, scr + o_q, toff, n, nb, tg, ngroups, tres);
        else if (wide) k_lookup_wt<Key, 2, 64, 3, true, 20><<<g, 64, 0, s>>>(dx, scr + o_q, toff, n, nb, tg, ngroups, tres);
        else k_lookup_wt<Key, 1, 64, 3, false><<<g, 64, 0, s>>>(dx, scr + o_q, toff, n, nb, tg, ngroups, tres);
    }
    g_cuart_launches++;
    ktimer_end(h, s, ev0, ev1, n);
    k_tgather<KS><<<unsigned(tiles), kBucketThreads, 0, s>>>(tres, (const uint16_t*)(scr + o_pos), toff, nb, n, out);
    g_cuart_launches++;
    rc = cudaGetLastError() == cudaSuccess ? CUART_OK : CUART_ERR_CUDA;
    scratch_free(h, scr, s);
    return rc;
}

static constexpr uint64_t kBucketMin = uint64_t(1) << 22;   // below this the batch is too small to reorder

cuart_status launch_lookup(const cuart_index* h, uint32_t kind, const void* q, const uint8_t* lens, uint64_t n,
                                  uint64_t* out, cudaStream_t s, const SegOut* so) {
    if (n == 0) return CUART_OK;
    // AUTO: integer keys only — for byte strings (c4, Zipf) the 33-B key copies cost
    // more than the locality gains (measured 9.0 vs 10.6 G lookups/s).
    const bool bucket = h->prebucket == CUART_PREBUCKET_ON ? n >= kBucketTile
                      : h->prebucket == CUART_PREBUCKET_AUTO && n >= kBucketMin && kind != CUART_KEY_BYTES;
    if (bucket && n < (uint64_t(1) << 32)) {
        const bool tiled = h->bucket_form == CUART_BUCKET_TILE && !so && h->slice_lut != CUART_SLICE_ON;
        if (tiled && kind == CUART_KEY_U64) return launch_tiled<KeyU64>(h, q, lens, n, out, s);
        if (tiled && kind == CUART_KEY_U32) return launch_tiled<KeyU32>(h, q, lens, n, out, s);
        if (tiled && kind == CUART_KEY_BYTES) return launch_tiled<KeyBytes>(h, q, lens, n, out, s);
        switch (kind) {
        case CUART_KEY_U64: return launch_bucketed<KeyU64>(h, q, lens, n, out, s, so);
        case CUART_KEY_U32: return launch_bucketed<KeyU32>(h, q, lens, n, out, s, so);
        default: return launch_bucketed<KeyBytes>(h, q, lens, n, out, s, so);
        }
    }
    return launch_lookup_direct(h, kind, q, lens, n, out, s, so);
}

cuart_status launch_lookup_direct(const cuart_index* h, uint32_t kind, const void* q, const uint8_t* lens,
                                  uint64_t n, uint64_t* out, cudaStream_t s, const SegOut* so, bool bucketed) {
    const int grid = grid_for(h, n);
    const DevIndex& dx = bucketed ? h->dix_links : h->dix;
    if (so && bucketed && dx.walk_wide && h->policy == 5 && h->ilp > 1 &&
        (kind == CUART_KEY_U64 || kind == CUART_KEY_U32)) {   // fused return from the wide walk (multi-GPU owner)
        cudaEvent_t ev0, ev1;
        ktimer_begin(h, s, ev0, ev1);
        const unsigned g = unsigned((n + 127) / 128);
        if (kind == CUART_KEY_U64) k_lookup_wq<KeyU64, 5, 2, 64, true, 3><<<g, 64, 0, s>>>(dx, q, lens, n, nullptr, *so);
        else k_lookup_wq<KeyU32, 5, 2, 64, true, 3><<<g, 64, 0, s>>>(dx, q, lens, n, nullptr, *so);
        g_cuart_launches++;
        ktimer_end(h, s, ev0, ev1, n);
        CU_TRY(cudaGetLastError());
        return CUART_OK;
    }
    if (so) {                                          // fused return: the default policy only
        cudaEvent_t ev0, ev1;
        ktimer_begin(h, s, ev0, ev1);
        switch (kind) {
        case CUART_KEY_U64: k_lookup<KeyU64, 5, true><<<grid, 256, 0, s>>>(dx, q, lens, n, nullptr, *so); break;
        case CUART_KEY_U32: k_lookup<KeyU32, 5, true><<<grid, 256, 0, s>>>(dx, q, lens, n, nullptr, *so); break;
        default: k_lookup<KeyBytes, 5, true><<<grid, 256, 0, s>>>(dx, q, lens, n, nullptr, *so); break;
        }
        g_cuart_launches++;
        ktimer_end(h, s, ev0, ev1, n);
        CU_TRY(cudaGetLastError());
        return CUART_OK;
    }
    cudaEvent_t ev0, ev1;
    ktimer_begin(h, s, ev0, ev1);                      // per-launch k_lookup timing (cuart_kernel_timer)
    if (bucketed && dx.walk_wide && h->policy == 5 && h->ilp > 1 && (kind == CUART_KEY_U64 || kind == CUART_KEY_U32)) {
        const unsigned tpb = h->wq_tpb == 32 || h->wq_tpb == 128 || h->wq_tpb == 256 ? h->wq_tpb : 64u;
        const unsigned qpt = h->ilp == 4 ? 4u : h->ilp == 3 ? 3u : 2u;   // queries per thread (template Q)
        const unsigned g = unsigned((n + tpb * qpt - 1) / (tpb * qpt));
#define CUART_WQ_Q(K, Q)                                                                          \
        if (tpb == 64 && h->wq_lp == 0) k_lookup_wq<K, 5, Q, 64, false, 0><<<g, 64, 0, s>>>(dx, q, lens, n, out); \
        else if (tpb == 64 && h->wq_lp == 1) k_lookup_wq<K, 5, Q, 64, false, 1><<<g, 64, 0, s>>>(dx, q, lens, n, out); \
        else if (tpb == 64 && h->wq_lp == 2) k_lookup_wq<K, 5, Q, 64, false, 2><<<g, 64, 0, s>>>(dx, q, lens, n, out); \
        else if (tpb == 64) k_lookup_wq<K, 5, Q, 64, false, 3><<<g, 64, 0, s>>>(dx, q, lens, n, out); \
        else if (tpb == 32) k_lookup_wq<K, 5, Q, 32, false, 3><<<g, 32, 0, s>>>(dx, q, lens, n, out); \
        else if (tpb == 128) k_lookup_wq<K, 5, Q, 128, false, 3><<<g, 128, 0, s>>>(dx, q, lens, n, out); \
        else k_lookup_wq<K, 5, Q, 256, false, 3><<<g, 256, 0, s>>>(dx, q, lens, n, out);
#define CUART_WQ(K)                                                                               \
        if (qpt == 4) { CUART_WQ_Q(K, 4) } else if (qpt == 3) { CUART_WQ_Q(K, 3) } else { CUART_WQ_Q(K, 2) }
        if (kind == CUART_KEY_U64) { CUART_WQ(KeyU64) } else { CUART_WQ(KeyU32) }
#undef CUART_WQ
#undef CUART_WQ_Q
        g_cuart_launches++;
        ktimer_end(h, s, ev0, ev1, n);
        CU_TRY(cudaGetLastError());
        return CUART_OK;
    }
    const unsigned ltpb = h->lk_tpb == 64 || h->lk_tpb == 128 ? h->lk_tpb : 256u;
    const unsigned lgrid = ltpb == 256 ? unsigned(grid) : unsigned((n + ltpb - 1) / ltpb);
#define CUART_LOOKUP(K, P)                                                                      \
    if (ltpb == 64) k_lookup<K, P, false, 64><<<lgrid, 64, 0, s>>>(dx, q, lens, n, out);        \
    else if (ltpb == 128) k_lookup<K, P, false, 128><<<lgrid, 128, 0, s>>>(dx, q, lens, n, out); \
    else k_lookup<K, P><<<grid, 256, 0, s>>>(dx, q, lens, n, out)
#define CUART_LOOKUP_POL(K)                          \
    switch (h->policy) {                             \
    case 0: CUART_LOOKUP(K, 0); break;               \
    case 2: CUART_LOOKUP(K, 2); break;               \
    case 3: CUART_LOOKUP(K, 3); break;               \
    case 4: CUART_LOOKUP(K, 4); break;               \
    case 5: CUART_LOOKUP(K, 5); break;               \
    case 1: CUART_LOOKUP(K, 1); break;               \
    default: CUART_LOOKUP(K, 5); break;              \
    }
    switch (kind) {
    case CUART_KEY_U64: CUART_LOOKUP_POL(KeyU64); break;
    case CUART_KEY_U32: CUART_LOOKUP_POL(KeyU32); break;
    default: CUART_LOOKUP_POL(KeyBytes); break;
    }
#undef CUART_LOOKUP_POL
#undef CUART_LOOKUP
    g_cuart_launches++;
    ktimer_end(h, s, ev0, ev1, n);
    CU_TRY(cudaGetLastError());
    return CUART_OK;
}

cuart_status scratch_alloc(const cuart_index* h, void** p, size_t bytes, cudaStream_t s) {
    *p = nullptr;
    if (bytes == 0) bytes = 256;
    const cudaError_t e = h->pool ? cudaMallocFromPoolAsync(p, bytes, h->pool, s) : cudaMallocAsync(p, bytes, s);
    if (e != cudaSuccess) {
        cudaGetLastError();
        *p = nullptr;
        return e == cudaErrorMemoryAllocation ? CUART_ERR_OOM : CUART_ERR_CUDA;
    }
    return CUART_OK;
}

void scratch_free(const cuart_index*, void* p, cudaStream_t s) {
    if (p) cudaFreeAsync(p, s);
}

cuart_status next_epoch(cuart_index* h, cudaStream_t s) {
    if (++h->epoch == 0xFFFFFFFFu) {        // epoch wrap: clear the conflict words
#if CUART_COLOCATED_WINNER
        k_clear_winners<<<h->num_sms * 8, 256, 0, s>>>(h->dix, h->count[5], h->count[6], h->count[7]);
        g_cuart_launches++;
        CU_TRY(cudaGetLastError());
#else
        if (h->total_leaves) CU_TRY(cudaMemsetAsync(h->dix.winner, 0, h->total_leaves * 8, s));
#endif
        h->epoch = 1;
    }
    return CUART_OK;
}

static constexpr uint64_t kUpdateChunk = uint64_t(1) << 30;   // op index must fit the low 32 bits

static cuart_status update_chunk(cuart_index* h, const DevIndex& dx, uint32_t kind, const void* k, const uint8_t* lens,
                                 const uint64_t* vals, const uint8_t* is_delete, int mode, uint64_t base, uint64_t m,
                                 cudaStream_t s, const uint32_t* opidx, bool bucketed, uint64_t* leafref,
                                 uint64_t* slotref) {
    const bool del = mode != 0;
    {
        const uint64_t epoch_hi = uint64_t(h->epoch) << 32;
        const int grid = grid_for(h, m);
        const size_t kstride = kind == CUART_KEY_U64 ? 8 : kind == CUART_KEY_U32 ? 4 : 32;
        const void* kb = (const uint8_t*)k + base * kstride;
        const uint8_t* lb = lens ? lens + base : nullptr;
        const uint64_t* vb = vals ? vals + base : nullptr;
        const uint8_t* db = (mode == 1) ? is_delete + base : nullptr;
        const uint32_t* ib = opidx ? opidx + base : nullptr;
#define CUART_UPD1(K, P, D) k_upd1<K, P, D><<<grid, 256, 0, s>>>(dx, kb, lb, vb, db, m, epoch_hi, leafref, slotref, ib)
#define CUART_UPD1_POL(K)                                    \
    if (h->policy == 0) {                                    \
        if (del) CUART_UPD1(K, 0, true); else CUART_UPD1(K, 0, false); \
    } else {                                                 \
        if (del) CUART_UPD1(K, 5, true); else CUART_UPD1(K, 5, false); \
    }
        const bool wq = !del && bucketed && dx.walk_wide && h->policy == 5 && h->ilp > 1 &&
                        (kind == CUART_KEY_U64 || kind == CUART_KEY_U32);
        const unsigned gq = unsigned((m + 128 - 1) / 128);         // 64 threads x 2 ops per CTA
        if (wq && kind == CUART_KEY_U64) k_upd1_wq<KeyU64, 2><<<gq, 64, 0, s>>>(dx, kb, vb, m, epoch_hi, leafref, ib);
        else if (wq) k_upd1_wq<KeyU32, 2><<<gq, 64, 0, s>>>(dx, kb, vb, m, epoch_hi, leafref, ib);
        else switch (kind) {
        case CUART_KEY_U64: CUART_UPD1_POL(KeyU64); break;
        case CUART_KEY_U32: CUART_UPD1_POL(KeyU32); break;
        case CUART_KEY_LONG: CUART_UPD1_POL(KeyLong); break;
        default: CUART_UPD1_POL(KeyBytes); break;
        }
#undef CUART_UPD1_POL
#undef CUART_UPD1
        g_cuart_launches++;
        CU_TRY(cudaGetLastError());
        if (del) k_upd2<true><<<grid, 256, 0, s>>>(dx, vb, db, m, epoch_hi, leafref, slotref, ib);
        else if (h->upd2_tpb == 64) k_upd2<false, 64><<<unsigned((m + 63) / 64), 64, 0, s>>>(dx, vb, nullptr, m, epoch_hi, leafref, nullptr, ib);
        else k_upd2<false><<<grid, 256, 0, s>>>(dx, vb, nullptr, m, epoch_hi, leafref, nullptr, ib);
        g_cuart_launches++;
        CU_TRY(cudaGetLastError());
    }
    return CUART_OK;
}

// mode: 0 = updates only, 1 = mixed (is_delete[i]), 2 = all deletes (vals unused).
// opidx: original op index of each op (pre-bucketed batches), or nullptr (= position).
cuart_status launch_update(cuart_index* h, uint32_t kind, const void* k, const uint8_t* lens,
                           const uint64_t* vals, const uint8_t* is_delete, int mode, uint64_t n,
                           cudaStream_t s, const uint32_t* opidx, bool bucketed, uint64_t* keep_leafref) {
    const bool del = mode != 0;
    const DevIndex& dx = bucketed ? h->dix_links : h->dix;
    const uint64_t cap = n < kUpdateChunk ? n : kUpdateChunk;
    uint64_t* leafref = keep_leafref;
    uint64_t* slotref = nullptr;
    cuart_status rc = CUART_OK;
    if (!leafref) rc = scratch_alloc(h, (void**)&leafref, cap * 8, s);
    if (rc == CUART_OK && del) rc = scratch_alloc(h, (void**)&slotref, cap * 8, s);
    for (uint64_t base = 0; base < n && rc == CUART_OK; base += kUpdateChunk) {
        const uint64_t m = (n - base) < kUpdateChunk ? (n - base) : kUpdateChunk;
        if (!h->hold_epoch && (rc = next_epoch(h, s)) != CUART_OK) break;
        rc = update_chunk(h, dx, kind, k, lens, vals, is_delete, mode, base, m, s, opidx, bucketed,
                          keep_leafref ? keep_leafref + base : leafref, slotref);
    }
    if (!keep_leafref) scratch_free(h, leafref, s);
    scratch_free(h, slotref, s);
    return rc;
}

// Pre-bucketed update batch (a5 applied to stage 1/2): ops are reordered by bucket
// together with their values and ORIGINAL op indices, which stay the priorities
// of the conflict resolution; no inverse permutation is needed because
// updates return nothing.
template <class Key>
static cuart_status launch_update_bucketed(cuart_index* h, const void* k, const uint8_t* lens, const uint64_t* vals,
                                          uint64_t n, cudaStream_t s) {
    const size_t ks = Key::kKind == 2 ? 8 : Key::kKind == 1 ? 4 : 32;
    auto al = [](size_t x) { return (x + 255) & ~size_t(255); };
    const uint64_t tiles = (n + kBucketTile - 1) / kBucketTile;
    const size_t o_hist = 0, o_tot = al(hist_entries(tiles) * 4), o_q = o_tot + 2048, o_len = o_q + al(n * ks),
                 o_val = o_len + al(Key::kKind == 3 ? n : 0), o_idx = o_val + al(n * 8), total = o_idx + al(n * 4);
    uint8_t* scr = nullptr;
    cuart_status rc = scratch_alloc(h, (void**)&scr, total, s);
    if (rc != CUART_OK) return rc;
    unsigned int* hist = (unsigned int*)(scr + o_hist);
    unsigned int* tot = (unsigned int*)(scr + o_tot);
    const uint32_t depth = (link_type(h->root) >= T_N4 && link_type(h->root) <= T_N256 ? link_aux(h->root) : 0u) |
                           (h->bucket_shift << 8);
    if ((uintptr_t(k) & 15) == 0) k_bhist<Key, true><<<unsigned(tiles), kBucketThreads, 0, s>>>(k, lens, n, ByteBucket(depth), hist);
    else k_bhist<Key, false><<<unsigned(tiles), kBucketThreads, 0, s>>>(k, lens, n, ByteBucket(depth), hist);
    k_bscan_rows<<<kBuckets >> h->bucket_shift, kBucketThreads, 0, s>>>(hist, tiles, tot);   // rows in use only
    k_bscan<<<1, kBuckets, 0, s>>>(tot, kBuckets >> h->bucket_shift);
    k_bscatter<Key, true><<<unsigned(tiles), kBucketThreads, bscatter_smem<Key, true>(), s>>>(
        k, lens, n, ByteBucket(depth), hist, tot, scr + o_q, Key::kKind == 3 ? scr + o_len : nullptr, nullptr, vals,
        (uint64_t*)(scr + o_val), (uint32_t*)(scr + o_idx));
    g_cuart_launches += 4;
    rc = cudaGetLastError() == cudaSuccess ? CUART_OK : CUART_ERR_CUDA;
    if (rc == CUART_OK)
        rc = launch_update(h, Key::kKind, scr + o_q, Key::kKind == 3 ? scr + o_len : nullptr,
                           (const uint64_t*)(scr + o_val), nullptr, 0, n, s, (const uint32_t*)(scr + o_idx), true);
    scratch_free(h, scr, s);
    return rc;
}

cuart_status dispatch_update(cuart_index* h, const void* k, const uint8_t* lens, const uint64_t* vals, uint64_t n,
                                    cudaStream_t s) {
    const bool bucket = h->prebucket == CUART_PREBUCKET_ON ? n >= kBucketTile
                      : h->prebucket == CUART_PREBUCKET_AUTO && n >= kBucketMin && h->key_kind != CUART_KEY_BYTES;
    if (bucket && n < kUpdateChunk) {
        switch (h->key_kind) {
        case CUART_KEY_U64: return launch_update_bucketed<KeyU64>(h, k, lens, vals, n, s);
        case CUART_KEY_U32: return launch_update_bucketed<KeyU32>(h, k, lens, vals, n, s);
        default: return launch_update_bucketed<KeyBytes>(h, k, lens, vals, n, s);
        }
    }
    return launch_update(h, h->key_kind, k, lens, vals, nullptr, 0, n, s);
}

// l2_persist: the caller's stream carries the persisting window for the launches of
// one call, then gets its previous policy back (attributes are captured per launch).
struct L2Window {
    cudaStream_t s = nullptr;
    bool set = false;
    cudaStreamAttrValue old{};
    L2Window(const cuart_index* h, cudaStream_t st) : s(st) {
        if (!h->l2_bytes) return;
        if (cudaStreamGetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &old) != cudaSuccess) {
            cudaGetLastError();
            return;
        }
        cudaStreamAttrValue v{};
        v.accessPolicyWindow.base_ptr = h->l2_base;
        v.accessPolicyWindow.num_bytes = h->l2_bytes;
        v.accessPolicyWindow.hitRatio = h->l2_hit;
        v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        set = cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v) == cudaSuccess;
        if (!set) cudaGetLastError();
    }
    ~L2Window() {
        if (set) cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &old);
    }
};

// ============================================================================ C ABI
extern "C" {

const char* cuart_status_string(cuart_status s) {
    switch (s) {
    case CUART_OK: return "ok";
    case CUART_ERR_INVALID_ARGUMENT: return "invalid argument";
    case CUART_ERR_KEY_LENGTH: return "key length must be 1..32";
    case CUART_ERR_NOT_PREFIX_FREE: return "key set is not prefix-free";
    case CUART_ERR_RESERVED_VALUE: return "value is the reserved CUART_MISS";
    case CUART_ERR_OOM: return "out of memory";
    case CUART_ERR_CUDA: return "CUDA error";
    case CUART_ERR_NCCL: return "NCCL error";
    case CUART_ERR_NO_DEVICE: return "no CUDA device";
    case CUART_ERR_TOO_LARGE: return "node buffer exceeds the link index range";
    case CUART_ERR_INTERNAL: return "internal error";
    }
    return "unknown status";
}

uint64_t cuart_launch_count(void) { return g_cuart_launches.load(); }

cuart_status cuart_layout_build(const cuart_keys* keys, const uint64_t* values, size_t n,
                                const cuart_build_opts* opts, cuart_layout** out) {
    if (!out || (!keys && n > 0)) return CUART_ERR_INVALID_ARGUMENT;
    *out = nullptr;
    uint32_t lut = opts ? opts->lut_bytes : 0;
    const uint32_t kind = keys ? uint32_t(keys->kind) : uint32_t(CUART_KEY_U64);
    if (lut == CUART_LUT_AUTO) lut = (kind == CUART_KEY_BYTES) ? 0 : (n >= (1u << 22) ? 3 : 0);
    cuart_layout* l = new (std::nothrow) cuart_layout();
    if (!l) return CUART_ERR_OOM;
    int rc;
    try {
        rc = build_host_layout(kind, keys ? keys->data : nullptr, keys ? keys->lengths : nullptr, values, n, lut, l->L);
    } catch (const std::bad_alloc&) {
        rc = CUART_ERR_OOM;
    } catch (...) {
        rc = CUART_ERR_INTERNAL;
    }
    if (rc != CUART_OK) {
        delete l;
        return cuart_status(rc);
    }
    *out = l;
    return CUART_OK;
}

cuart_status cuart_layout_free(cuart_layout* l) {
    delete l;
    return CUART_OK;
}

cuart_status cuart_layout_view_get(const cuart_layout* l, cuart_layout_view* v) {
    if (!l || !v) return CUART_ERR_INVALID_ARGUMENT;
    memset(v, 0, sizeof(*v));
    for (int t = 1; t < 8; t++) {
        v->buf[t] = l->L.buf[t].data();
        v->count[t] = l->L.count[t];
        v->record_bytes[t] = record_bytes(t);
    }
    v->lut = l->L.lut.empty() ? nullptr : l->L.lut.data();
    v->lut_entries = l->L.lut.size();
    v->root = l->L.root;
    v->lut_bytes = l->L.lut_bytes;
    v->key_kind = l->L.key_kind;
    v->n_keys = l->L.n_keys;
    return CUART_OK;
}

cuart_status cuart_layout_lookup(const cuart_layout* l, const cuart_keys* q, size_t n, uint64_t* out, int threads) {
    if (!l || !q || (n > 0 && (!q->data || !out))) return CUART_ERR_INVALID_ARGUMENT;
    if (uint32_t(q->kind) != l->L.key_kind) return CUART_ERR_INVALID_ARGUMENT;
    if (q->kind == CUART_KEY_BYTES && n > 0 && !q->lengths) return CUART_ERR_INVALID_ARGUMENT;
    host_layout_lookup(l->L, l->L.key_kind, q->data, q->lengths, n, out, threads);
    return CUART_OK;
}

cuart_status cuart_layout_sectors_ex(const cuart_layout* l, const cuart_keys* q, size_t n, uint32_t* sectors,
                                     int threads, uint32_t flags) {
    if (!l || !q || (n > 0 && (!q->data || !sectors))) return CUART_ERR_INVALID_ARGUMENT;
    if (q->kind == CUART_KEY_BYTES && n > 0 && !q->lengths) return CUART_ERR_INVALID_ARGUMENT;
    if (uint32_t(q->kind) != l->L.key_kind) return CUART_ERR_INVALID_ARGUMENT;
    host_layout_sectors(l->L, l->L.key_kind, q->data, q->lengths, n, sectors, threads,
                        (flags & CUART_SECTORS_WIDE) && !l->L.lut.empty(), (flags >> 8) & 0xFFu);
    return CUART_OK;
}

cuart_status cuart_layout_sectors(const cuart_layout* l, const cuart_keys* q, size_t n, uint32_t* sectors, int threads) {
    if (!l || !q || (n > 0 && (!q->data || !sectors))) return CUART_ERR_INVALID_ARGUMENT;
    if (uint32_t(q->kind) != l->L.key_kind) return CUART_ERR_INVALID_ARGUMENT;
    if (q->kind == CUART_KEY_BYTES && n > 0 && !q->lengths) return CUART_ERR_INVALID_ARGUMENT;
    host_layout_sectors(l->L, l->L.key_kind, q->data, q->lengths, n, sectors, threads);
    return CUART_OK;
}

// Compact 32-bit LUT (kernels.cuh expand_lut32): integer keys only, every entry must fit.
static bool compact_lut(const HostLayout& L, std::vector<uint32_t>& out) {
    if (L.lut.empty() || L.key_kind == CUART_KEY_BYTES) return false;
    out.resize(L.lut.size());
    for (size_t i = 0; i < L.lut.size(); i++) {
        const uint64_t l = L.lut[i];
        const uint32_t t = link_type(l);
        const uint64_t idx = link_index(l);
        if (t == T_NULL) { out[i] = 0; continue; }
        if (t >= T_LEAF8) {
            if (idx > 0x1FFFFFFFull) return false;
            out[i] = (t << 29) | uint32_t(idx);
        } else {
            const uint32_t rel = link_aux(l) - L.lut_bytes;
            if (link_aux(l) < L.lut_bytes || rel > 6 || idx > 0x3FFFFFFull) return false;
            out[i] = (t << 29) | (rel << 26) | uint32_t(idx);
        }
    }
    return true;
}

static uint64_t expand_lut32_host(uint32_t e, uint32_t k, uint32_t leaf_len) {
    const uint32_t t = e >> 29;
    if (t == T_NULL) return 0;
    if (t >= T_LEAF8) return make_link(t, leaf_len, e & 0x1FFFFFFFu);
    return make_link(t, k + ((e >> 26) & 7u), e & 0x3FFFFFFu);
}

// Rank LUT (kernels.cuh expand_lut_rank): 32-entry blocks of 32 B —
//   u32 plane[3] (type code bits of each entry), u32 exc (entry lives in the 64-bit
//   link table), u32 base[4] (index of the first N4 / N16 / N48 / N256 entry).
// An inner-node entry is encoded in the block when its branch depth is k and its
// index is base[type] + (number of earlier entries of that type in the block).
// Leaves (lexicographically numbered, so not consecutive) and everything else are
// exceptions read from the full 64-bit table.  Integer keys only.
// ---- skip table (byte strings; kernels.cuh skip_start) -----------------------
// The node covering every key with the D-byte prefix P: walk from the root table (or
// the root) following P's bytes until a leaf or an inner node branching at depth >= D.
static uint64_t skip_cover(const HostLayout& L, const uint8_t* P, uint32_t D) {
    uint64_t link = L.root;
    if (L.lut_bytes && D >= L.lut_bytes && !L.lut.empty()) {
        uint64_t p = 0;
        for (uint32_t b = 0; b < L.lut_bytes; b++) p = (p << 8) | P[b];
        link = L.lut[p];
    }
    for (;;) {
        const uint32_t t = link_type(link), aux = link_aux(link);
        if (t == T_NULL || t >= T_LEAF8 || aux >= D) return link;
        const uint8_t* rec = L.buf[t].data() + link_index(link) * record_bytes(t);
        const uint32_t b = P[aux];
        uint64_t child = 0;
        if (t == T_N4 || t == T_N16) {
            const uint8_t* keys = rec + (t == T_N4 ? kN4Keys : kN16Keys);
            const int nk = t == T_N4 ? 4 : 16;
            int c = -1;
            for (int i = 0; i < nk; i++)
                if (keys[i] == b) {
                    c = i;
                    break;
                }
            if (c < 0) return 0;
            memcpy(&child, rec + (t == T_N4 ? kN4Child : kN16Child) + 8 * c, 8);
        } else if (t == T_N48) {
            const uint8_t s = rec[kN48Index + b];
            if (s == kN48Empty) return 0;
            memcpy(&child, rec + kN48Child + 8 * s, 8);
        } else {
            memcpy(&child, rec + kN256Child + 8 * b, 8);
        }
        link = child;
    }
}

// D = the largest prefix length in [lut_bytes + 2, 16] whose distinct prefixes (an
// upper bound: counted per leaf class, each sorted) number at most 2^18, so the
// table (2 slots per prefix, 32 B each: <= 16 MB) stays L2-resident.  Returns false
// (no table) for integer keys or when no such D exists.
static bool build_skip_table(const HostLayout& L, std::vector<uint64_t>& tab, uint32_t& D, uint64_t& mask,
                             uint32_t max_log2) {
    if (L.key_kind != CUART_KEY_BYTES || L.root == 0) return false;
    uint64_t cnt[17] = {0};
    for (int t = T_LEAF8; t <= T_LEAF32; t++) {
        const uint64_t m = L.count[t];
        const uint32_t kb = kLeafKeyBytes[t];
        for (uint64_t i = 0; i < m; i++) {
            const uint8_t* k = L.buf[t].data() + i * record_bytes(t);
            const uint32_t len = L.leaf_len[t].empty() ? kb : L.leaf_len[t][i];
            uint32_t lcp = 0, plen = 0;
            if (i > 0) {
                const uint8_t* pk = k - record_bytes(t);
                plen = L.leaf_len[t].empty() ? kb : L.leaf_len[t][i - 1];
                while (lcp < 16 && lcp < kb && pk[lcp] == k[lcp]) lcp++;
            }
            for (uint32_t d = 1; d <= 16 && d <= len; d++)
                if (i == 0 || lcp < d || plen < d) cnt[d]++;
        }
    }
    D = 0;
    for (uint32_t d = 16; d >= L.lut_bytes + 2 && d >= 2; d--)
        if (cnt[d] > 0 && cnt[d] <= (uint64_t(1) << max_log2)) {
            D = d;
            break;
        }
    if (D == 0) return false;
    uint64_t slots = 1;
    while (slots < 2 * cnt[D]) slots <<= 1;
    mask = slots - 1;
    tab.assign(slots * 4, 0);
    for (int t = T_LEAF8; t <= T_LEAF32; t++) {
        const uint64_t m = L.count[t];
        const uint32_t kb = kLeafKeyBytes[t];
        for (uint64_t i = 0; i < m; i++) {
            const uint8_t* k = L.buf[t].data() + i * record_bytes(t);
            const uint32_t len = L.leaf_len[t].empty() ? kb : L.leaf_len[t][i];
            if (len < D) continue;
            uint8_t P[16] = {0};
            memcpy(P, k, D < kb ? D : kb);
            uint64_t p0, p1;
            memcpy(&p0, P, 8);
            memcpy(&p1, P + 8, 8);
            p0 &= low_bytes_mask(D < 8 ? D : 8u);
            p1 = D > 8 ? p1 & low_bytes_mask(D - 8) : 0ull;
            uint64_t h = skip_hash(p0, p1) & mask;
            bool present = false;
            while (tab[4 * h + 2] != 0) {
                if (tab[4 * h] == p0 && tab[4 * h + 1] == p1) {
                    present = true;
                    break;
                }
                h = (h + 1) & mask;
            }
            if (present) continue;
            const uint64_t link = skip_cover(L, P, D);
            if (link == 0) continue;                       // cannot happen for a stored key
            tab[4 * h] = p0;
            tab[4 * h + 1] = p1;
            tab[4 * h + 2] = link;
        }
    }
    return true;
}

static bool rank_lut(const HostLayout& L, std::vector<uint64_t>& blocks, uint64_t& n_exc) {
    if (L.lut.empty() || L.key_kind == CUART_KEY_BYTES) return false;
    const uint32_t k = L.lut_bytes;
    const uint64_t nb = (L.lut.size() + 31) / 32;
    blocks.assign(nb * 4, 0);
    n_exc = 0;
    for (uint64_t bi = 0; bi < nb; bi++) {
        uint32_t plane[3] = {0, 0, 0}, exc = 0, base[5] = {0, 0, 0, 0, 0};
        uint64_t cnt[5] = {0};
        for (uint32_t j = 0; j < 32 && bi * 32 + j < L.lut.size(); j++) {
            const uint64_t l = L.lut[bi * 32 + j];
            const uint32_t t = link_type(l);
            if (t == T_NULL) continue;
            const uint64_t idx = link_index(l);
            bool ok = t <= T_N256 && link_aux(l) == k;
            if (ok && cnt[t] == 0) {
                if (idx > 0xFFFFFFFFull) ok = false;
                else base[t] = uint32_t(idx);
            }
            if (ok && idx != uint64_t(base[t]) + cnt[t]) ok = false;
            if (!ok) {
                exc |= 1u << j;
                n_exc++;
                continue;
            }
            cnt[t]++;
            for (int pb = 0; pb < 3; pb++)
                if (t & (1u << pb)) plane[pb] |= 1u << j;
        }
        uint32_t* blk = reinterpret_cast<uint32_t*>(&blocks[bi * 4]);
        blk[0] = plane[0];
        blk[1] = plane[1];
        blk[2] = plane[2];
        blk[3] = exc;
        for (int t = 1; t <= 4; t++) blk[3 + t] = base[t];
    }
    return true;
}

cuart_status cuart_upload(const cuart_layout* lay, const cuart_build_opts* opts, cuart_index** out) {
    if (!lay || !out) return CUART_ERR_INVALID_ARGUMENT;
    *out = nullptr;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) return CUART_ERR_NO_DEVICE;
    int dev = (opts && opts->device >= 0) ? opts->device : -1;
    if (dev < 0) CU_TRY(cudaGetDevice(&dev));
    if (dev >= ndev) return CUART_ERR_NO_DEVICE;
    CU_TRY(cudaSetDevice(dev));
    const HostLayout& L = lay->L;
    cuart_index* h = new (std::nothrow) cuart_index();
    if (!h) return CUART_ERR_OOM;
    h->device = dev;
    cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, dev);
    h->key_kind = L.key_kind;
    h->lut_bytes = L.lut_bytes;
    h->long_bytes = L.long_bytes;
    h->long_off = L.long_off;
    h->long_vals = L.long_vals;
    h->root = L.root;
    h->n_keys = L.n_keys;
    h->max_depth = L.max_depth;
    // arena: [N4 | N16 | N48 | N256 | leaf8 | leaf16 | leaf32 | winner | LUT | err], 256-B aligned
    auto align = [](uint64_t x) { return (x + 255) & ~uint64_t(255); };
    uint64_t off = 0;
    for (int t = 1; t < 8; t++) {
        h->count[t] = L.count[t];
        h->off[t] = off;
        off = align(off + L.buf[t].size());
    }
    h->total_leaves = L.count[5] + L.count[6] + L.count[7];
    h->winner_off = off;
    if (!CUART_COLOCATED_WINNER) off = align(off + h->total_leaves * 8);
    h->free_off = off;
    off = align(off + 8 + h->total_leaves * 4);
    h->llen_off = off;                                 // BYTES: key length per leaf (range queries)
    if (L.key_kind == CUART_KEY_BYTES) off = align(off + h->total_leaves);
    std::vector<uint32_t> lut32;
    std::vector<uint64_t> lutr;
    uint32_t fmt = opts ? opts->lut_format : CUART_LUT_FORMAT_AUTO;
    if (L.lut.empty()) fmt = CUART_LUT_LINKS;
    if (fmt == CUART_LUT_FORMAT_AUTO) fmt = (L.key_kind >= CUART_KEY_BYTES) ? CUART_LUT_LINKS : CUART_LUT_RANK;
    if (L.key_kind == CUART_KEY_LONG) fmt = CUART_LUT_LINKS;
    if (fmt == CUART_LUT_RANK && !rank_lut(L, lutr, h->lut_exceptions)) fmt = CUART_LUT_LINKS;
    if (fmt == CUART_LUT_COMPACT32 && !compact_lut(L, lut32)) fmt = CUART_LUT_LINKS;
    if (fmt < CUART_LUT_LINKS || fmt > CUART_LUT_RANK) {
        delete h;
        return CUART_ERR_INVALID_ARGUMENT;
    }
    h->lut_format = fmt;
    if (const char* pe = getenv("CUART_POLICY")) h->policy = atoi(pe);
    // tuning knobs (environment; the defaults are the measured best)
    if (const char* pe = getenv("CUART_GRID_CTAS_PER_SM")) h->grid_ctas_per_sm = atoi(pe);
    if (const char* pe = getenv("CUART_ILP")) h->ilp = atoi(pe);
    if (const char* pe = getenv("CUART_WQ_TPB")) h->wq_tpb = unsigned(atoi(pe));
    if (const char* pe = getenv("CUART_LOOKUP_TPB")) h->lk_tpb = unsigned(atoi(pe));
    if (const char* pe = getenv("CUART_UPD2_TPB")) h->upd2_tpb = unsigned(atoi(pe));
    if (const char* pe = getenv("CUART_WQ_LEAFPOL")) h->wq_lp = atoi(pe);
    h->prebucket = opts ? opts->prebucket : CUART_PREBUCKET_AUTO;
    if (h->prebucket > CUART_PREBUCKET_ON) {
        delete h;
        return CUART_ERR_INVALID_ARGUMENT;
    }
    if (const char* pe = getenv("CUART_PREBUCKET")) h->prebucket = atoi(pe) ? CUART_PREBUCKET_ON : CUART_PREBUCKET_OFF;
    {
        const uint32_t bf = opts ? opts->bucket_form : CUART_BUCKET_FORM_AUTO;
        if (bf > CUART_BUCKET_TILE) {
            delete h;
            return CUART_ERR_INVALID_ARGUMENT;
        }
        h->bucket_form = bf == CUART_BUCKET_GLOBAL ? CUART_BUCKET_GLOBAL : CUART_BUCKET_TILE;
        if (const char* pe = getenv("CUART_WT_MINB")) h->wt_minb = uint32_t(atoi(pe));
        if (const char* pe = getenv("CUART_WT_TPB")) h->wt_tpb = uint32_t(atoi(pe));
        if (const char* pe = getenv("CUART_TSORT_VEC")) h->tsort_vec = uint32_t(atoi(pe));
        if (const char* pe = getenv("CUART_TSORT_B1K")) h->tsort_b1k = uint32_t(atoi(pe));
        if (const char* pe = getenv("CUART_TILE_GROUP")) {
            const int v = atoi(pe);
            h->tile_group = v < 1 ? 1u : v > 64 ? 64u : uint32_t(v);
        }
        if (const char* pe = getenv("CUART_BUCKET_FORM")) h->bucket_form = atoi(pe) == 1 ? CUART_BUCKET_GLOBAL : CUART_BUCKET_TILE;
    }
    cudaFuncSetAttribute(k_bscatter<KeyU64>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(bscatter_smem<KeyU64>()));
    cudaFuncSetAttribute(k_bscatter<KeyU32>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(bscatter_smem<KeyU32>()));
    cudaFuncSetAttribute(k_bscatter<KeyBytes>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         int(bscatter_smem<KeyBytes>()));
    cudaFuncSetAttribute(k_bscatter<KeyU64, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         int(bscatter_smem<KeyU64, true>()));
    cudaFuncSetAttribute(k_bscatter<KeyU32, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         int(bscatter_smem<KeyU32, true>()));
    cudaFuncSetAttribute(k_bscatter<KeyBytes, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         int(bscatter_smem<KeyBytes, true>()));
    // LUT region: 64-bit links (LINKS, and the exception table of RANK) then the compact form
    h->lut_off = off;
    const bool need_links = fmt == CUART_LUT_LINKS || fmt == CUART_LUT_RANK;
    if (need_links) off = align(off + L.lut.size() * 8);
    h->lutc_off = off;
    off = align(off + lut32.size() * 4 + lutr.size() * 8);
    // wide root table for the pre-bucketed walks (kernels.cuh start_wide)
    // Worth it when most table entries lead to an N4/N16 (c3: 92%): a 32-B entry costs
    // the L2 like the N4 block / N16 keys it saves, but more than an 8-B LINKS entry,
    // so for N48/N256 targets (c2, c5) the walk keeps the LINKS table (measured on c2:
    // 2.45 ms LINKS vs 2.94 ms wide per 2^28; c3: 14.38 ms LINKS vs 11.12 ms wide per 2^30).
    h->wide = false;
    if (need_links && !L.lut.empty()) {
        uint64_t small = 0, nonnull = 0;
        for (uint64_t l : L.lut) {
            nonnull += l != 0;
            small += link_type(l) == T_N4 || link_type(l) == T_N16 ||
                     (link_type(l) == T_N256 && leaf_run_link(L.buf[T_N256].data() + link_index(l) * record_bytes(T_N256), T_N256));
        }
        h->wide = nonnull > 0 && 2 * small >= nonnull;
    }
    uint32_t wide_opt = opts ? opts->wide_lut : CUART_WIDE_AUTO;
    if (const char* pe = getenv("CUART_WIDE")) wide_opt = uint32_t(atoi(pe));
    if (wide_opt > CUART_WIDE_ON) {
        delete h;
        return CUART_ERR_INVALID_ARGUMENT;
    }
    if (wide_opt == CUART_WIDE_OFF) h->wide = false;
    if (wide_opt == CUART_WIDE_ON) h->wide = need_links && !L.lut.empty();
    std::vector<uint64_t> lutw;
    if (h->wide) {
        lutw.assign(L.lut.size() * 4, 0);
        for (size_t p = 0; p < L.lut.size(); p++) {
            const uint64_t l = L.lut[p];
            lutw[4 * p] = l;
            const uint32_t t = link_type(l);
            if (t != T_N4 && t != T_N16 && t != T_N256) continue;
            const uint8_t* rec = L.buf[t].data() + link_index(l) * record_bytes(t);
            if (t == T_N256) {                            // full N256 of leaves: child b = run + b
                lutw[4 * p + 3] = leaf_run_link(rec, t);
                continue;
            }
            uint8_t keys16[16];
            if (t == T_N4) {                              // padded to 16 with the last key, like an N16,
                memcpy(keys16, rec + kN4Keys, 4);         // so the walk searches both the same way
                memset(keys16 + 4, rec[kN4Keys + 3], 12);
            } else {
                memcpy(keys16, rec + kN16Keys, 16);
            }
            memcpy(&lutw[4 * p + 1], keys16, 16);
            lutw[4 * p + 3] = leaf_run_link(rec, t);      // child i = run + i when all children are leaves
        }
    }
    h->lutw_off = off;
    off = align(off + lutw.size() * 8);
    std::vector<uint64_t> skipt;
    uint32_t skip_d = 0;
    uint64_t skip_mask = 0;
    {
        const char* pe = getenv("CUART_SKIP");
        uint32_t lg = opts && opts->skip_log2 ? opts->skip_log2 : 20u;
        if (const char* pl = getenv("CUART_SKIP_LOG2")) lg = uint32_t(atoi(pl));
        lg = lg > 26 ? 26u : lg;
        if (!(pe && atoi(pe) == 0)) build_skip_table(L, skipt, skip_d, skip_mask, lg);
    }
    h->skip_off = off;
    off = align(off + skipt.size() * 8);
    h->err_off = off;
    off = align(off + 256);
    h->arena_bytes = off;
    {
        uint64_t walked = lutw.size() * 8;                // records a bucketed walk reads
        for (int t = 1; t < 8; t++) walked += L.buf[t].size();
        h->bucket_shift = walked <= (uint64_t(64) << 26) ? 2u : 0u;   // slice <= 64 MB at 64 buckets
        if (const char* pe = getenv("CUART_BUCKET_SHIFT")) h->bucket_shift = uint32_t(atoi(pe)) & 7u;
    }
    cudaError_t e = cudaMalloc(&h->arena, off);
    if (e != cudaSuccess) {
        delete h;
        return e == cudaErrorMemoryAllocation ? CUART_ERR_OOM : CUART_ERR_CUDA;
    }
    cuart_status rc = CUART_OK;
    for (int t = 1; t < 8 && rc == CUART_OK; t++)
        if (!L.buf[t].empty() && cudaMemcpy(h->arena + h->off[t], L.buf[t].data(), L.buf[t].size(), cudaMemcpyHostToDevice) != cudaSuccess)
            rc = CUART_ERR_CUDA;
    if (rc == CUART_OK && need_links && !L.lut.empty() &&
        cudaMemcpy(h->arena + h->lut_off, L.lut.data(), L.lut.size() * 8, cudaMemcpyHostToDevice) != cudaSuccess)
        rc = CUART_ERR_CUDA;
    if (rc == CUART_OK && !lut32.empty() &&
        cudaMemcpy(h->arena + h->lutc_off, lut32.data(), lut32.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess)
        rc = CUART_ERR_CUDA;
    if (rc == CUART_OK && !lutr.empty() &&
        cudaMemcpy(h->arena + h->lutc_off, lutr.data(), lutr.size() * 8, cudaMemcpyHostToDevice) != cudaSuccess)
        rc = CUART_ERR_CUDA;
    if (rc == CUART_OK && !skipt.empty() &&
        cudaMemcpy(h->arena + h->skip_off, skipt.data(), skipt.size() * 8, cudaMemcpyHostToDevice) != cudaSuccess)
        rc = CUART_ERR_CUDA;
    if (rc == CUART_OK && !lutw.empty() &&
        cudaMemcpy(h->arena + h->lutw_off, lutw.data(), lutw.size() * 8, cudaMemcpyHostToDevice) != cudaSuccess)
        rc = CUART_ERR_CUDA;
    if (rc == CUART_OK && !CUART_COLOCATED_WINNER && h->total_leaves &&
        cudaMemset(h->arena + h->winner_off, 0, h->total_leaves * 8) != cudaSuccess)
        rc = CUART_ERR_CUDA;
    if (rc == CUART_OK && cudaMemset(h->arena + h->err_off, 0, 256) != cudaSuccess) rc = CUART_ERR_CUDA;
    if (rc == CUART_OK && cudaMemset(h->arena + h->free_off, 0, 8) != cudaSuccess) rc = CUART_ERR_CUDA;
    if (L.key_kind == CUART_KEY_BYTES)
        for (int t = T_LEAF8, o = 0; t <= T_LEAF32 && rc == CUART_OK; o += int(L.count[t]), t++)
            if (L.count[t] && cudaMemcpy(h->arena + h->llen_off + o, L.leaf_len[t].data(), L.count[t],
                                         cudaMemcpyHostToDevice) != cudaSuccess)
                rc = CUART_ERR_CUDA;
    if (rc != CUART_OK) {
        cudaFree(h->arena);
        delete h;
        return rc;
    }
    // k_lookup_slice geometry: bucket byte = root branch depth d; the slice of bucket b
    // is the table entries of prefix C.b.* (C = the d-byte common prefix, read off the
    // first non-null entry), 256^(k-1-d) entries = 1 B each in RANK form.
    h->slice_lut = opts ? opts->slice_lut : CUART_SLICE_AUTO;
    if (h->slice_lut > CUART_SLICE_ON) rc = CUART_ERR_INVALID_ARGUMENT;
    if (const char* pe = getenv("CUART_SLICE")) h->slice_lut = atoi(pe) == 1 ? CUART_SLICE_OFF : atoi(pe) == 2 ? CUART_SLICE_ON : CUART_SLICE_AUTO;
    if (h->slice_lut == CUART_SLICE_ON) h->bucket_shift = 0;    // the slice walk needs one bucket per root byte
    {
        const uint32_t rt = link_type(L.root);
        const uint32_t d = (rt >= T_N4 && rt <= T_N256) ? link_aux(L.root) : 0xFFu;
        const uint32_t k = L.lut_bytes;
        if (fmt == CUART_LUT_RANK && L.key_kind != CUART_KEY_BYTES && d != 0xFFu && d + 2 <= k && !L.lut.empty()) {
            uint64_t p0 = 0;
            while (p0 < L.lut.size() && L.lut[p0] == 0) p0++;
            if (p0 < L.lut.size()) {
                h->slice_shift = 8 * (k - 1 - d);
                h->slice_e0 = (p0 >> (8 * (k - d))) << (8 * (k - d));
                const int smem = 1 << h->slice_shift;
                int occ = 0;
                if (cudaFuncSetAttribute(k_lookup_slice<KeyU64, 5>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) == cudaSuccess &&
                    cudaFuncSetAttribute(k_lookup_slice<KeyU32, 5>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) == cudaSuccess &&
                    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, L.key_kind == CUART_KEY_U64
                                                                            ? (const void*)k_lookup_slice<KeyU64, 5>
                                                                            : (const void*)k_lookup_slice<KeyU32, 5>,
                                                                  kSliceThreads, smem) == cudaSuccess && occ > 0) {
                    h->slice_grid = occ * h->num_sms;
                    h->slice_ok = true;
                }
            }
        }
    }
    if (rc != CUART_OK) {
        cudaFree(h->arena);
        delete h;
        return rc;
    }
    DevIndex& d = h->dix;
    for (int t = 1; t < 8; t++) d.base[t] = h->arena + h->off[t];
    d.base[0] = nullptr;
    d.root = L.root;
    d.lut = need_links ? (const uint64_t*)(h->arena + h->lut_off) : nullptr;
    d.lut32 = lut32.empty() ? nullptr : (const uint32_t*)(h->arena + h->lutc_off);
    d.lutr = lutr.empty() ? nullptr : (const uint4*)(h->arena + h->lutc_off);
    d.lut_bytes = L.lut_bytes;
    d.fixed_len = L.key_kind == CUART_KEY_U64 ? 8 : L.key_kind == CUART_KEY_U32 ? 4 : 0;
    d.key_kind = L.key_kind;
    d.winner = CUART_COLOCATED_WINNER ? nullptr : (uint64_t*)(h->arena + h->winner_off);
    d.leaf_base[5] = 0;
    d.leaf_base[6] = L.count[5];
    d.leaf_base[7] = L.count[5] + L.count[6];
    d.err = (uint32_t*)(h->arena + h->err_off);
    d.free_count = (unsigned long long*)(h->arena + h->free_off);
    d.free_list = (uint32_t*)(h->arena + h->free_off + 8);
    // Pre-bucketed walks read the LINKS table (present for RANK as its exception
    // table): with the batch bucketed the bucket's slice of it is L2-resident, and an
    // 8-B request costs the L2 less than the 32-B rank block (K-GATHER: 245 vs 145 G
    // random requests/s); measured -4% walk time on c3 and c2.
    d.lutw = h->wide ? (uint64_t*)(h->arena + h->lutw_off) : nullptr;
    d.lut_entries = L.lut.size();
    d.walk_wide = 0;
    d.skip = skipt.empty() ? nullptr : (const uint64_t*)(h->arena + h->skip_off);
    d.skip_mask = skip_mask;
    d.skip_d = skip_d;
    h->skip_d = skip_d;
    h->skip_entries = skipt.size() / 4;
    h->dix_links = d;
    if (d.lut) {
        h->dix_links.lutr = nullptr;
        h->dix_links.lut32 = nullptr;
        h->dix_links.walk_wide = h->wide ? 1u : 0u;
    }
    {   // the index's own pool for stream-ordered scratch: it keeps its memory mapped
        // between calls (no re-mapping per batch) and is destroyed with the index, so
        // other allocators (PyTorch's caching allocator, the device default pool) never
        // see memory held on the index's behalf
        cudaMemPoolProps pp = {};
        pp.allocType = cudaMemAllocationTypePinned;
        pp.location.type = cudaMemLocationTypeDevice;
        pp.location.id = dev;
        if (cudaMemPoolCreate(&h->pool, &pp) == cudaSuccess) {
            uint64_t keep = ~uint64_t(0);
            cudaMemPoolSetAttribute(h->pool, cudaMemPoolAttrReleaseThreshold, &keep);
        } else {
            cudaGetLastError();
            h->pool = nullptr;
        }
    }
    if (opts && opts->l2_persist && h->lutw_off + lutw.size() * 8 > h->lut_off) {
        // the root tables the walks start from (LINKS + compact/rank + wide), contiguous in
        // the arena: persisting lines up to the device's persisting-L2 limit
        int maxp = 0, maxw = 0;
        cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, dev);
        cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxAccessPolicyWindowSize, dev);
        const size_t span = h->lutw_off + lutw.size() * 8 - h->lut_off;
        if (maxp > 0 && maxw > 0) {
            h->l2_base = h->arena + h->lut_off;
            h->l2_bytes = span < size_t(maxw) ? span : size_t(maxw);
            h->l2_hit = float(maxp) >= float(h->l2_bytes) ? 1.f : float(maxp) / float(h->l2_bytes);
            if (cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, size_t(maxp)) != cudaSuccess) {
                cudaGetLastError();
                h->l2_bytes = 0;
            }
        }
    }
    *out = h;
    return CUART_OK;
}

cuart_status cuart_build(const cuart_keys* keys, const uint64_t* values, size_t n, const cuart_build_opts* opts,
                         cuart_index** out) {
    if (!out) return CUART_ERR_INVALID_ARGUMENT;
    *out = nullptr;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) return CUART_ERR_NO_DEVICE;
    cuart_layout* l = nullptr;
    cuart_status rc = cuart_layout_build(keys, values, n, opts, &l);
    if (rc != CUART_OK) return rc;
    rc = cuart_upload(l, opts, out);
    cuart_layout_free(l);
    return rc;
}

cuart_status cuart_destroy(cuart_index* h) {
    if (!h) return CUART_OK;
    cudaSetDevice(h->device);
    if (h->dist) dist_teardown(h);        // collective: every rank of the group destroys together
    cudaDeviceSynchronize();
    cudaFree(h->arena);
    drop_kevents(h);
    for (int i = 0; i < kStages; i++) {
        if (h->stage[i]) cudaFree(h->stage[i]);
        if (h->stage_out[i]) cudaFree(h->stage_out[i]);
        if (h->stage_len[i]) cudaFree(h->stage_len[i]);
        if (h->stage_val[i]) cudaFree(h->stage_val[i]);
        if (h->streams[i]) cudaStreamDestroy(h->streams[i]);
        if (h->ev_copied[i]) cudaEventDestroy(h->ev_copied[i]);
        if (h->ev_free[i]) cudaEventDestroy(h->ev_free[i]);
    }
    if (h->ustream) cudaStreamDestroy(h->ustream);
    if (h->ev_join) cudaEventDestroy(h->ev_join);
    if (h->pool) cudaMemPoolDestroy(h->pool);   // every scratch block was freed in stream order
    delete h;
    return CUART_OK;
}

// ---------------------------------------------------------------- f4: long keys
cuart_status cuart_build_long(const uint8_t* data, const uint64_t* offsets, const uint64_t* values, size_t n,
                              const cuart_build_opts* opts, cuart_index** out) {
    if (!out || (n > 0 && (!data || !offsets || !values))) return CUART_ERR_INVALID_ARGUMENT;
    *out = nullptr;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) return CUART_ERR_NO_DEVICE;
    uint32_t lut = opts ? opts->lut_bytes : 0;
    if (lut == CUART_LUT_AUTO) lut = 0;
    cuart_layout* l = new (std::nothrow) cuart_layout();
    if (!l) return CUART_ERR_OOM;
    int rc;
    try {
        rc = build_host_layout(CUART_KEY_LONG, data, nullptr, values, n, lut, l->L, offsets);
    } catch (const std::bad_alloc&) {
        rc = CUART_ERR_OOM;
    }
    if (rc == CUART_OK) rc = cuart_upload(l, opts, out);
    cuart_layout_free(l);
    return cuart_status(rc);
}

// Upload a packed host batch (data, offsets) to fresh device buffers on stream s.
static cuart_status upload_long_batch(const uint8_t* data, const uint64_t* offsets, size_t n, cudaStream_t s,
                                      uint8_t** dq, uint64_t** doff) {
    const uint64_t nb = offsets[n];
    CU_TRY(cudaMallocAsync((void**)dq, nb ? nb : 1, s));
    CU_TRY(cudaMallocAsync((void**)doff, (n + 1) * 8, s));
    CU_TRY(cudaMemcpyAsync(*dq, data, nb, cudaMemcpyHostToDevice, s));
    CU_TRY(cudaMemcpyAsync(*doff, offsets, (n + 1) * 8, cudaMemcpyHostToDevice, s));
    return CUART_OK;
}

static bool long_key_equal(const cuart_index* h, uint64_t idx, const uint8_t* key, uint64_t len) {
    const uint64_t a = h->long_off[idx], b = h->long_off[idx + 1];
    return b - a == len && memcmp(h->long_bytes.data() + a, key, len) == 0;
}

static cuart_status check_long_batch(const cuart_index* h, const uint8_t* data, const uint64_t* offsets, size_t n) {
    if (!h || h->key_kind != CUART_KEY_LONG) return CUART_ERR_INVALID_ARGUMENT;
    if (n > 0 && (!data || !offsets)) return CUART_ERR_INVALID_ARGUMENT;
    if (n >= (uint64_t(1) << 30)) return CUART_ERR_INVALID_ARGUMENT;
    for (size_t i = 0; i < n; i++) {
        if (offsets[i + 1] < offsets[i]) return CUART_ERR_INVALID_ARGUMENT;
        const uint64_t l = offsets[i + 1] - offsets[i];
        if (l == 0 || l > kMaxLongKey) return CUART_ERR_KEY_LENGTH;
    }
    return CUART_OK;
}

cuart_status cuart_lookup_long(cuart_index* h, const uint8_t* data, const uint64_t* offsets, size_t n, uint64_t* out,
                               void* stream) {
    cuart_status rc = check_long_batch(h, data, offsets, n);
    if (rc != CUART_OK) return rc;
    if (n == 0) return CUART_OK;
    if (!out) return CUART_ERR_INVALID_ARGUMENT;
    CU_TRY(cudaSetDevice(h->device));
    cudaStream_t s = (cudaStream_t)stream;
    uint8_t* dq = nullptr;
    uint64_t* doff = nullptr;
    if ((rc = upload_long_batch(data, offsets, n, s, &dq, &doff)) != CUART_OK) return rc;
    uint64_t* dout = nullptr;
    uint8_t* dsig = nullptr;
    CU_TRY(cudaMallocAsync((void**)&dout, n * 8, s));
    CU_TRY(cudaMallocAsync((void**)&dsig, n, s));
    k_lookup_long<5><<<grid_for(h, n), 256, 0, s>>>(h->dix, dq, doff, n, dout, dsig);
    g_cuart_launches++;
    CU_TRY(cudaGetLastError());
    std::vector<uint8_t> sig(n);
    CU_TRY(cudaMemcpyAsync(out, dout, n * 8, cudaMemcpyDeviceToHost, s));
    CU_TRY(cudaMemcpyAsync(sig.data(), dsig, n, cudaMemcpyDeviceToHost, s));
    CU_TRY(cudaFreeAsync(dq, s));
    CU_TRY(cudaFreeAsync(doff, s));
    CU_TRY(cudaFreeAsync(dout, s));
    CU_TRY(cudaFreeAsync(dsig, s));
    CU_TRY(cudaStreamSynchronize(s));
    // the host side of P:126 option 2: full-key compare against the host leaf
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < int64_t(n); i++) {
        if (!sig[i]) continue;
        const uint64_t idx = out[i];
        out[i] = long_key_equal(h, idx, data + offsets[i], offsets[i + 1] - offsets[i]) ? h->long_vals[idx] : kMiss;
    }
    return CUART_OK;
}

cuart_status cuart_update_long(cuart_index* h, const uint8_t* data, const uint64_t* offsets, const uint64_t* values,
                               size_t n, void* stream) {
    cuart_status rc = check_long_batch(h, data, offsets, n);
    if (rc != CUART_OK) return rc;
    if (n == 0) return CUART_OK;
    if (!values) return CUART_ERR_INVALID_ARGUMENT;
    CU_TRY(cudaSetDevice(h->device));
    cudaStream_t s = (cudaStream_t)stream;
    uint8_t* dq = nullptr;
    uint64_t* doff = nullptr;
    if ((rc = upload_long_batch(data, offsets, n, s, &dq, &doff)) != CUART_OK) return rc;
    uint64_t* dval = nullptr;
    uint64_t* dref = nullptr;
    CU_TRY(cudaMallocAsync((void**)&dval, n * 8, s));
    CU_TRY(cudaMallocAsync((void**)&dref, n * 8, s));
    CU_TRY(cudaMemcpyAsync(dval, values, n * 8, cudaMemcpyHostToDevice, s));
    // device leaves: the two-stage kernels; host leaves: stage 1 leaves their links in dref
    rc = launch_update(h, CUART_KEY_LONG, dq, (const uint8_t*)doff, dval, nullptr, 0, n, s, nullptr, false, dref);
    std::vector<uint64_t> ref(n);
    if (rc == CUART_OK && cudaMemcpyAsync(ref.data(), dref, n * 8, cudaMemcpyDeviceToHost, s) != cudaSuccess)
        rc = CUART_ERR_CUDA;
    cudaFreeAsync(dq, s);
    cudaFreeAsync(doff, s);
    cudaFreeAsync(dval, s);
    cudaFreeAsync(dref, s);
    CU_TRY(cudaStreamSynchronize(s));
    if (rc != CUART_OK) return rc;
    // host leaves in op order: sequential semantics, the last op on a key wins
    for (size_t i = 0; i < n; i++) {
        const uint64_t l = ref[i];
        if (!l || link_type(l) != T_LEAF_HOST) continue;
        const uint64_t idx = link_index(l);
        if (long_key_equal(h, idx, data + offsets[i], offsets[i + 1] - offsets[i])) h->long_vals[idx] = values[i];
    }
    return CUART_OK;
}

cuart_status cuart_lookup(const cuart_index* h, const cuart_keys* q, size_t n, uint64_t* out, void* stream) {
    cuart_status rc = check_keys(h, q, n);
    if (rc != CUART_OK) return rc;
    if (n == 0) return CUART_OK;
    if (!out) return CUART_ERR_INVALID_ARGUMENT;
    L2Window w(h, (cudaStream_t)stream);
    return launch_lookup(h, h->key_kind, q->data, q->lengths, n, out, (cudaStream_t)stream);
}

cuart_status cuart_update(cuart_index* h, const cuart_keys* k, const uint64_t* v, size_t n, void* stream) {
    cuart_status rc = check_keys(h, k, n);
    if (rc != CUART_OK) return rc;
    if (n == 0) return CUART_OK;
    if (!v) return CUART_ERR_INVALID_ARGUMENT;
    L2Window w(h, (cudaStream_t)stream);
    return dispatch_update(h, k->data, k->lengths, v, n, (cudaStream_t)stream);
}

cuart_status cuart_update_ex(cuart_index* h, const cuart_keys* k, const uint64_t* v, const uint8_t* is_delete, size_t n,
                             void* stream) {
    cuart_status rc = check_keys(h, k, n);
    if (rc != CUART_OK) return rc;
    if (n == 0) return CUART_OK;
    if (!v || !is_delete) return CUART_ERR_INVALID_ARGUMENT;
    return launch_update(h, h->key_kind, k->data, k->lengths, v, is_delete, 1, n, (cudaStream_t)stream);
}

cuart_status cuart_erase(cuart_index* h, const cuart_keys* k, size_t n, void* stream) {
    cuart_status rc = check_keys(h, k, n);
    if (rc != CUART_OK) return rc;
    if (n == 0) return CUART_OK;
    return launch_update(h, h->key_kind, k->data, k->lengths, nullptr, nullptr, 2, n, (cudaStream_t)stream);
}

cuart_status cuart_range_leaf8(const uint8_t* leaves, uint64_t nleaves, uint32_t kind, const void* lo, const void* hi,
                               size_t n, uint64_t* bounds, void* stream);   // route.cu

cuart_status cuart_range_bytes(const uint8_t* const* rec, const uint8_t* const* len, const uint64_t* count,
                               const uint8_t* lo, const uint8_t* llo, const uint8_t* hi, const uint8_t* lhi, size_t n,
                               uint64_t* bounds, void* stream);   // route.cu

cuart_status cuart_range(const cuart_index* h, const cuart_keys* lo, const cuart_keys* hi, size_t n, uint64_t* bounds,
                         void* stream) {
    cuart_status rc = check_keys(h, lo, n);
    if (rc == CUART_OK) rc = check_keys(h, hi, n);
    if (rc != CUART_OK) return rc;
    if (n == 0) return CUART_OK;
    if (!bounds) return CUART_ERR_INVALID_ARGUMENT;
    if (h->key_kind == CUART_KEY_BYTES) {
        const uint8_t* rec[3];
        const uint8_t* len[3];
        const uint64_t cnt[3] = {h->count[T_LEAF8], h->count[T_LEAF16], h->count[T_LEAF32]};
        for (int c = 0; c < 3; c++) {
            rec[c] = h->dix.base[T_LEAF8 + c];
            len[c] = h->arena + h->llen_off + h->dix.leaf_base[T_LEAF8 + c];
        }
        return cuart_range_bytes(rec, len, cnt, (const uint8_t*)lo->data, lo->lengths, (const uint8_t*)hi->data,
                                 hi->lengths, n, bounds, stream);
    }
    return cuart_range_leaf8(h->dix.base[T_LEAF8], h->count[T_LEAF8], h->key_kind, lo->data, hi->data, n, bounds,
                             stream);
}

cuart_status cuart_kernel_timer(cuart_index* h, int enable) {
    if (!h) return CUART_ERR_INVALID_ARGUMENT;
    std::lock_guard<std::mutex> g(h->kmu);
    drop_kevents(h);
    h->ktimer = enable != 0;
    return CUART_OK;
}

cuart_status cuart_kernel_time(cuart_index* h, double* total_ms, uint64_t* launches, uint64_t* lookups) {
    uint64_t sl = 0;
    return cuart_kernel_time_ex(h, total_ms, launches, lookups, &sl);
}

cuart_status cuart_kernel_time_ex(cuart_index* h, double* total_ms, uint64_t* launches, uint64_t* lookups,
                                  uint64_t* slice_launches) {
    if (!h || !total_ms || !launches || !lookups || !slice_launches) return CUART_ERR_INVALID_ARGUMENT;
    std::lock_guard<std::mutex> g(h->kmu);
    double t = 0;
    for (auto& e : h->kev) {
        float ms = 0;
        CU_TRY(cudaEventSynchronize(e.second));
        CU_TRY(cudaEventElapsedTime(&ms, e.first, e.second));
        t += ms;
    }
    *total_ms = t;
    *launches = h->kev.size();
    *lookups = h->klookups;
    *slice_launches = h->kslice;
    drop_kevents(h);
    return CUART_OK;
}

cuart_status cuart_debug_set_epoch(cuart_index* h, uint32_t epoch) {
    if (!h || epoch == 0 || epoch == 0xFFFFFFFFu) return CUART_ERR_INVALID_ARGUMENT;
    CU_TRY(cudaSetDevice(h->device));
    CU_TRY(cudaDeviceSynchronize());
    h->epoch = epoch;
    return CUART_OK;
}

cuart_status cuart_free_leaves(const cuart_index* h, uint32_t* ids, size_t cap, size_t* count) {
    if (!h || !count) return CUART_ERR_INVALID_ARGUMENT;
    CU_TRY(cudaSetDevice(h->device));
    CU_TRY(cudaDeviceSynchronize());
    unsigned long long c = 0;
    CU_TRY(cudaMemcpy(&c, h->dix.free_count, 8, cudaMemcpyDeviceToHost));
    *count = size_t(c);
    if (ids && cap) {
        const size_t m = size_t(c) < cap ? size_t(c) : cap;
        if (m) CU_TRY(cudaMemcpy(ids, h->dix.free_list, m * 4, cudaMemcpyDeviceToHost));
    }
    return CUART_OK;
}

// ---------------------------------------------------------------- host-buffer pipelines

static size_t key_stride(uint32_t kind);
static size_t stage_chunk();
static cuart_status ensure_stage(cuart_index* h) {
    if (h->stage_cap) return CUART_OK;
    const size_t c = stage_chunk(), ks = key_stride(h->key_kind);
    for (int i = 0; i < kStages; i++) {
        CU_TRY(cudaMalloc(&h->stage[i], c * ks));
        CU_TRY(cudaMalloc(&h->stage_out[i], c * 8));
        if (h->key_kind == CUART_KEY_BYTES) CU_TRY(cudaMalloc(&h->stage_len[i], c));
        CU_TRY(cudaMalloc(&h->stage_val[i], c * 8));
        CU_TRY(cudaStreamCreateWithFlags(&h->streams[i], cudaStreamNonBlocking));
        CU_TRY(cudaEventCreateWithFlags(&h->ev_copied[i], cudaEventDisableTiming));
        CU_TRY(cudaEventCreateWithFlags(&h->ev_free[i], cudaEventDisableTiming));
    }
    CU_TRY(cudaStreamCreateWithFlags(&h->ustream, cudaStreamNonBlocking));
    h->stage_cap = c;
    return CUART_OK;
}

static size_t key_stride(uint32_t kind) { return kind == CUART_KEY_U64 ? 8 : kind == CUART_KEY_U32 ? 4 : 32; }

// The host pipelines run on the index's own non-blocking streams, which do not
// synchronise with the legacy default stream: order them after every operation
// already queued there (and, through the legacy stream's implicit synchronisation,
// on every blocking stream), e.g. a cuart_update(h, ..., NULL) just before.
static cuart_status join_legacy_stream(cuart_index* h) {
    if (!h->ev_join) CU_TRY(cudaEventCreateWithFlags(&h->ev_join, cudaEventDisableTiming));
    CU_TRY(cudaEventRecord(h->ev_join, 0));
    for (int i = 0; i < kStages; i++) CU_TRY(cudaStreamWaitEvent(h->streams[i], h->ev_join, 0));
    CU_TRY(cudaStreamWaitEvent(h->ustream, h->ev_join, 0));
    return CUART_OK;
}
// ops per host-pipeline chunk: kStageChunk, or CUART_STAGE_CHUNK read when the
// handle's staging buffers are first allocated (a tuning / test knob)
static size_t stage_chunk() {
    size_t v = kStageChunk;
    if (const char* pe = getenv("CUART_STAGE_CHUNK")) v = size_t(strtoull(pe, nullptr, 0));
    return v == 0 || v > (size_t(1) << 28) ? kStageChunk : v;
}

cuart_status cuart_lookup_host(const cuart_index* hc, const cuart_keys* q, size_t n, uint64_t* out) {
    cuart_index* h = const_cast<cuart_index*>(hc);
    cuart_status rc = check_keys(h, q, n);
    if (rc != CUART_OK) return rc;
    if (n == 0) return CUART_OK;
    if (!out) return CUART_ERR_INVALID_ARGUMENT;
    CU_TRY(cudaSetDevice(h->device));
    if ((rc = ensure_stage(h)) != CUART_OK) return rc;
    if ((rc = join_legacy_stream(h)) != CUART_OK) return rc;
    const size_t ks = key_stride(h->key_kind);
    size_t c = 0;
    const size_t chunk = h->stage_cap;
    for (size_t base = 0; base < n; base += chunk, c++) {
        const size_t m = (n - base) < chunk ? (n - base) : chunk;
        const int s = int(c % kStages);
        cudaStream_t st = h->streams[s];
        CU_TRY(cudaMemcpyAsync(h->stage[s], (const uint8_t*)q->data + base * ks, m * ks, cudaMemcpyHostToDevice, st));
        if (h->key_kind == CUART_KEY_BYTES) CU_TRY(cudaMemcpyAsync(h->stage_len[s], q->lengths + base, m, cudaMemcpyHostToDevice, st));
        rc = launch_lookup(h, h->key_kind, h->stage[s], h->key_kind == CUART_KEY_BYTES ? h->stage_len[s] : nullptr, m, h->stage_out[s], st);
        if (rc != CUART_OK) return rc;
        CU_TRY(cudaMemcpyAsync(out + base, h->stage_out[s], m * 8, cudaMemcpyDeviceToHost, st));
    }
    for (int i = 0; i < kStages; i++) CU_TRY(cudaStreamSynchronize(h->streams[i]));
    return CUART_OK;
}

cuart_status cuart_update_host(cuart_index* h, const cuart_keys* k, const uint64_t* v, size_t n) {
    cuart_status rc = check_keys(h, k, n);
    if (rc != CUART_OK) return rc;
    if (n == 0) return CUART_OK;
    if (!v) return CUART_ERR_INVALID_ARGUMENT;
    CU_TRY(cudaSetDevice(h->device));
    if ((rc = ensure_stage(h)) != CUART_OK) return rc;
    if ((rc = join_legacy_stream(h)) != CUART_OK) return rc;
    const size_t ks = key_stride(h->key_kind);
    // The kernels of all chunks run in op order on ONE stream (sequential semantics
    // across chunks); the H2D copies of the next chunks run on the staging sets' own
    // streams and overlap them (events: set filled -> kernels; kernels done -> set free).
    cudaStream_t ust = h->ustream;
    size_t c = 0;
    const size_t chunk = h->stage_cap;
    for (size_t base = 0; base < n; base += chunk, c++) {
        const size_t m = (n - base) < chunk ? (n - base) : chunk;
        const int s = int(c % kStages);
        cudaStream_t cst = h->streams[s];
        if (c >= size_t(kStages)) CU_TRY(cudaStreamWaitEvent(cst, h->ev_free[s], 0));
        CU_TRY(cudaMemcpyAsync(h->stage[s], (const uint8_t*)k->data + base * ks, m * ks, cudaMemcpyHostToDevice, cst));
        if (h->key_kind == CUART_KEY_BYTES) CU_TRY(cudaMemcpyAsync(h->stage_len[s], k->lengths + base, m, cudaMemcpyHostToDevice, cst));
        CU_TRY(cudaMemcpyAsync(h->stage_val[s], v + base, m * 8, cudaMemcpyHostToDevice, cst));
        CU_TRY(cudaEventRecord(h->ev_copied[s], cst));
        CU_TRY(cudaStreamWaitEvent(ust, h->ev_copied[s], 0));
        rc = dispatch_update(h, h->stage[s], h->key_kind == CUART_KEY_BYTES ? h->stage_len[s] : nullptr, h->stage_val[s], m, ust);
        if (rc != CUART_OK) return rc;
        CU_TRY(cudaEventRecord(h->ev_free[s], ust));
    }
    CU_TRY(cudaStreamSynchronize(ust));
    return CUART_OK;
}

// ---------------------------------------------------------------- introspection
cuart_status cuart_stats(const cuart_index* h, cuart_stats_t* s) {
    if (!h || !s) return CUART_ERR_INVALID_ARGUMENT;
    memset(s, 0, sizeof(*s));
    for (int t = 1; t < 8; t++) {
        s->count[t] = h->count[t];
        s->bytes[t] = h->count[t] * record_bytes(t);
    }
    s->n_keys = h->n_keys;
    s->lut_bytes = h->lut_bytes;
    s->lut_entries = h->lut_bytes ? (uint64_t(1) << (8 * h->lut_bytes)) : 0;
    s->lut_bytes_total = h->lut_format == CUART_LUT_COMPACT32 ? s->lut_entries * 4
                       : h->lut_format == CUART_LUT_RANK ? s->lut_entries * 9 : s->lut_entries * 8;
    if (h->wide) s->lut_bytes_total += s->lut_entries * 32;       // wide table of the bucketed walks
    s->lut_format = h->lut_format;
    s->lut_exceptions = h->lut_exceptions;
    s->wide_lut = h->wide ? 1u : 0u;
    s->l2_window_bytes = h->l2_bytes;
    s->skip_prefix = h->skip_d;
    s->skip_slots = h->skip_entries;
    s->arena_bytes = h->arena_bytes;
    s->key_kind = h->key_kind;
    s->root = h->root;
    s->max_depth = h->max_depth;
    return CUART_OK;
}

cuart_status cuart_dump(const cuart_index* h, cuart_layout** out) {
    if (!h || !out) return CUART_ERR_INVALID_ARGUMENT;
    *out = nullptr;
    CU_TRY(cudaSetDevice(h->device));
    CU_TRY(cudaDeviceSynchronize());
    cuart_layout* l = new (std::nothrow) cuart_layout();
    if (!l) return CUART_ERR_OOM;
    HostLayout& L = l->L;
    L.key_kind = h->key_kind;
    L.root = h->root;
    L.lut_bytes = h->lut_bytes;
    L.n_keys = h->n_keys;
    L.max_depth = h->max_depth;
    try {
        for (int t = 1; t < 8; t++) {
            L.count[t] = h->count[t];
            L.buf[t].resize(h->count[t] * record_bytes(t));
            if (!L.buf[t].empty() &&
                cudaMemcpy(L.buf[t].data(), h->arena + h->off[t], L.buf[t].size(), cudaMemcpyDeviceToHost) != cudaSuccess) {
                delete l;
                return CUART_ERR_CUDA;
            }
        }
        if (h->lut_bytes) {
            L.lut.resize(uint64_t(1) << (8 * h->lut_bytes));
            if (h->lut_format == CUART_LUT_COMPACT32) {
                std::vector<uint32_t> c(L.lut.size());
                if (cudaMemcpy(c.data(), h->arena + h->lutc_off, c.size() * 4, cudaMemcpyDeviceToHost) != cudaSuccess) {
                    delete l;
                    return CUART_ERR_CUDA;
                }
                for (size_t i = 0; i < c.size(); i++) L.lut[i] = expand_lut32_host(c[i], h->lut_bytes, h->dix.fixed_len);
            } else if (cudaMemcpy(L.lut.data(), h->arena + h->lut_off, L.lut.size() * 8, cudaMemcpyDeviceToHost) != cudaSuccess) {
                delete l;
                return CUART_ERR_CUDA;
            }
        }
    } catch (...) {
        delete l;
        return CUART_ERR_OOM;
    }
    *out = l;
    return CUART_OK;
}

cuart_status cuart_get_error(cuart_index* h) {
    if (!h) return CUART_ERR_INVALID_ARGUMENT;
    CU_TRY(cudaSetDevice(h->device));
    CU_TRY(cudaDeviceSynchronize());
    uint32_t flag = 0;
    CU_TRY(cudaMemcpy(&flag, h->dix.err, 4, cudaMemcpyDeviceToHost));
    if (flag) {
        CU_TRY(cudaMemset(h->dix.err, 0, 4));
        return CUART_ERR_RESERVED_VALUE;
    }
    return CUART_OK;
}

}  // extern "C"
