// kernels.cuh — device-side traversal of the CuART layout (sm_100a).
//
// Lookup algorithm of PAPER.md Fig. 3 within the type-segregated buffers
// (§3.2.1): decode the packed link (type in the MSBs, index in the LSBs),
// read a record of a size known before the request, search the child on the key
// byte, repeat; compare the full key at the leaf.  B200 reading: the branch depth
// rides in the link (layout.h), so no node header is read on the path, the
// compressed prefix is skipped optimistically and the leaf compare decides.
#pragma once
#include <stdint.h>

#include "layout.h"

namespace cuart {

struct DevIndex {
    const uint8_t* base[8];       // record buffers per type code
    uint64_t root;                // packed root link
    const uint64_t* lut;          // root lookup table, or nullptr
    const uint32_t* lut32;        // compact 32-bit root lookup table, or nullptr
    const uint4* lutr;            // rank-form root lookup table (64-B blocks), or nullptr
    uint32_t lut_bytes;
    uint32_t fixed_len;           // key length of integer kinds (4 / 8), 0 for byte strings
    uint32_t key_kind;
    uint64_t* winner;             // per-leaf conflict word for updates (global leaf id)
    uint64_t leaf_base[8];        // global leaf id = leaf_base[type] + index
    uint32_t* err;                // sticky device error flag
    uint32_t* free_list;          // freed leaf ids (global leaf id), capacity = #leaves
    unsigned long long* free_count;  // number of entries in free_list
    uint64_t* lutw;               // wide root table (32 B/entry: link + the target N4/N16's keys), or nullptr
    uint64_t lut_entries;         // 2^(8 lut_bytes)
    uint32_t walk_wide;           // 1: lookups start from lutw (pre-bucketed walks, whose lutw slice is L2-resident)
    // byte strings: skip table over the first skip_d key bytes (32-B entries {prefix
    // words p0, p1, link of the node covering that prefix, 0}, open addressing), or nullptr
    const uint64_t* skip;
    uint64_t skip_mask;
    uint32_t skip_d;
};

// Segmented output (multi-GPU fused return, §8(e)): result i goes to
// dst[s] + (i - start[s]) for the segment s with start[s] <= i < start[s + 1];
// dst[s] may be a peer GPU's window (CUDA IPC over NVLink), so the kernel that
// produces the results also performs the return transfer.
constexpr int kMaxSeg = 16;
struct SegOut {
    uint32_t nseg;
    uint64_t start[kMaxSeg + 1];
    uint64_t* dst[kMaxSeg];
    __device__ __forceinline__ uint64_t* at(uint64_t i) const {
        uint32_t s = 0;
#pragma unroll 1
        while (s + 1 < nseg && i >= start[s + 1]) s++;
        return dst[s] + (i - start[s]);
    }
};

// ----------------------------------------------------------------------------- loads
__device__ __forceinline__ uint64_t ld_nc_u64(const void* p) {
    uint64_t v;
    asm volatile("ld.global.nc.u64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ uint32_t ld_nc_u8(const void* p) {
    uint16_t v;
    asm volatile("ld.global.nc.u8 %0, [%1];" : "=h"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ uint4 ld_nc_v4(const void* p) {
    uint4 v;
    asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}
// 256-bit (32 B) load: one request on sm_100 (SASS LDG.E.ENL2.256); p 32-B aligned.
struct U8x32 { uint32_t w[8]; };
__device__ __forceinline__ U8x32 ld_nc_v8(const void* p) {
    U8x32 v;
    asm volatile("ld.global.nc.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(v.w[0]), "=r"(v.w[1]), "=r"(v.w[2]), "=r"(v.w[3]), "=r"(v.w[4]), "=r"(v.w[5]), "=r"(v.w[6]),
                   "=r"(v.w[7]) : "l"(p));
    return v;
}
// Leaf values are rewritten by the update kernels: read them through L2 (coherent path).
__device__ __forceinline__ uint64_t ld_cg_u64(const void* p) {
    uint64_t v;
    asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}

__device__ __forceinline__ uint64_t bswap64(uint64_t x) {
    uint32_t lo = uint32_t(x), hi = uint32_t(x >> 32);
    return (uint64_t(__byte_perm(lo, 0, 0x0123)) << 32) | __byte_perm(hi, 0, 0x0123);
}

// ----------------------------------------------------------------------------- key views
// U64: numeric key, canonical bytes are big-endian (reading C2).
struct KeyU64 {
    uint64_t k;
    static constexpr uint32_t kKind = 2;
    template <bool STREAM>
    __device__ __forceinline__ static KeyU64 load(const void* q, const uint8_t*, uint64_t i) {
        const unsigned long long* p = (const unsigned long long*)q + i;
        return KeyU64{STREAM ? uint64_t(__ldcs(p)) : uint64_t(*p)};
    }
    __device__ __forceinline__ uint32_t len() const { return 8; }
    __device__ __forceinline__ uint32_t byte(uint32_t d) const { return uint32_t(k >> (56 - 8 * d)) & 0xFF; }
    __device__ __forceinline__ uint64_t prefix(uint32_t nb) const { return k >> (64 - 8 * nb); }
    // One 16-byte load brings key and value of a leaf8 record.
    template <class LD>
    __device__ __forceinline__ bool leaf_match(const LD& ld, const uint8_t* rec, uint32_t t, uint32_t aux, uint64_t& val) const {
        const uint4 r = ld.leafv4(rec);
        val = uint64_t(r.z) | (uint64_t(r.w) << 32);
        return aux == 8 && (uint64_t(r.x) | (uint64_t(r.y) << 32)) == bswap64(k);
    }
};

struct KeyU32 {
    uint32_t k;
    static constexpr uint32_t kKind = 1;
    template <bool STREAM>
    __device__ __forceinline__ static KeyU32 load(const void* q, const uint8_t*, uint64_t i) {
        const unsigned int* p = (const unsigned int*)q + i;
        return KeyU32{STREAM ? uint32_t(__ldcs(p)) : uint32_t(*p)};
    }
    __device__ __forceinline__ uint32_t len() const { return 4; }
    __device__ __forceinline__ uint32_t byte(uint32_t d) const { return (k >> (24 - 8 * d)) & 0xFF; }
    __device__ __forceinline__ uint64_t prefix(uint32_t nb) const { return uint64_t(k) >> (32 - 8 * nb); }
    template <class LD>
    __device__ __forceinline__ bool leaf_match(const LD& ld, const uint8_t* rec, uint32_t t, uint32_t aux, uint64_t& val) const {
        const uint4 r = ld.leafv4(rec);
        val = uint64_t(r.z) | (uint64_t(r.w) << 32);
        return aux == 4 && r.y == 0 && r.x == __byte_perm(k, 0, 0x0123);
    }
};

// BYTES: 32-byte slot + length; bytes past the length are masked to zero.
struct KeyBytes {
    uint64_t w[4];   // little-endian words of the zero-padded slot
    uint32_t l;
    static constexpr uint32_t kKind = 3;
    template <bool STREAM>
    __device__ __forceinline__ static KeyBytes load(const void* q, const uint8_t* lens, uint64_t i) {
        KeyBytes kb;
        const uint4* pq = (const uint4*)q + 2 * i;
        const uint4 a = STREAM ? __ldcs(pq) : pq[0];
        const uint4 b = STREAM ? __ldcs(pq + 1) : pq[1];
        kb.w[0] = uint64_t(a.x) | (uint64_t(a.y) << 32);
        kb.w[1] = uint64_t(a.z) | (uint64_t(a.w) << 32);
        kb.w[2] = uint64_t(b.x) | (uint64_t(b.y) << 32);
        kb.w[3] = uint64_t(b.z) | (uint64_t(b.w) << 32);
        kb.l = lens[i];
#pragma unroll
        for (int j = 0; j < 4; j++) {
            const int lo = 8 * j;
            const int keep = int(kb.l) - lo;   // bytes of word j inside the key
            uint64_t m = keep >= 8 ? ~0ull : (keep <= 0 ? 0ull : ((1ull << (8 * keep)) - 1));
            kb.w[j] &= m;
        }
        return kb;
    }
    __device__ __forceinline__ uint32_t len() const { return l; }
    __device__ __forceinline__ uint64_t word(uint32_t j) const {
        return j == 0 ? w[0] : j == 1 ? w[1] : j == 2 ? w[2] : w[3];
    }
    __device__ __forceinline__ uint32_t byte(uint32_t d) const { return uint32_t(word(d >> 3) >> (8 * (d & 7))) & 0xFF; }
    __device__ __forceinline__ uint64_t prefix(uint32_t nb) const {
        uint64_t p = 0;
        for (uint32_t b = 0; b < nb; b++) p = (p << 8) | byte(b);
        return p;
    }
    // leaf8: one 16-B request.  leaf16 (32 B, 32-B aligned): one 256-bit request for
    // key + value.  leaf32 (48 B; 32-B aligned for even indices, 16 mod 32 for odd
    // ones): a 32-B and a 16-B request in the order the alignment allows, i.e. 2
    // requests instead of 3 (random L2 requests are what the walk is bound by, §5).
    template <class LD>
    __device__ __forceinline__ bool leaf_match(const LD& ld, const uint8_t* rec, uint32_t t, uint32_t aux, uint64_t& val) const {
        if (t == T_LEAF8) {
            const uint4 a = ld.leafv4(rec);
            val = uint64_t(a.z) | (uint64_t(a.w) << 32);
            return aux == l && (uint64_t(a.x) | (uint64_t(a.y) << 32)) == w[0];
        }
        if (t == T_LEAF16) {
            const U8x32 r = ld.leafv8(rec);
            val = uint64_t(r.w[4]) | (uint64_t(r.w[5]) << 32);
            return aux == l && (uint64_t(r.w[0]) | (uint64_t(r.w[1]) << 32)) == w[0] &&
                   (uint64_t(r.w[2]) | (uint64_t(r.w[3]) << 32)) == w[1];
        }
        const bool odd = (uintptr_t(rec) & 16) != 0;              // record index odd: rec = 16 mod 32
        const uint4 a = ld.leafv4(odd ? rec : rec + 32);           // odd: key[0,16)   even: value | conflict
        const U8x32 b = ld.leafv8(odd ? rec + 16 : rec);           // odd: key[16,32) | value | conflict   even: key[0,32)
        uint32_t k[8];
#pragma unroll
        for (int j = 0; j < 4; j++) {
            k[j] = odd ? (&a.x)[j] : b.w[j];
            k[4 + j] = odd ? b.w[j] : b.w[4 + j];
        }
        val = odd ? (uint64_t(b.w[4]) | (uint64_t(b.w[5]) << 32)) : (uint64_t(a.x) | (uint64_t(a.y) << 32));
        bool eq = aux == l;
#pragma unroll
        for (int j = 0; j < 4; j++) eq &= (uint64_t(k[2 * j]) | (uint64_t(k[2 * j + 1]) << 32)) == w[j];
        return eq;
    }
};

// f4 (CUART_KEY_LONG): a 1..255-byte key read in place from the packed query
// buffer (key i = q[off[i], off[i+1]); `lens` carries the offsets array).
struct KeyLong {
    const uint8_t* p;
    uint32_t l;
    static constexpr uint32_t kKind = 4;
    template <bool STREAM>
    __device__ __forceinline__ static KeyLong load(const void* q, const uint8_t* offs, uint64_t i) {
        const uint64_t* off = (const uint64_t*)offs;
        const uint64_t a = off[i], b = off[i + 1];
        return KeyLong{(const uint8_t*)q + a, uint32_t(b - a)};
    }
    __device__ __forceinline__ uint32_t len() const { return l; }
    __device__ __forceinline__ uint32_t byte(uint32_t d) const { return __ldg(p + d); }
    __device__ __forceinline__ uint64_t prefix(uint32_t nb) const {
        uint64_t v = 0;
        for (uint32_t b = 0; b < nb; b++) v = (v << 8) | byte(b);
        return v;
    }
    // device leaves hold keys of <= 32 bytes: equal length, then byte for byte
    template <class LD>
    __device__ __forceinline__ bool leaf_match(const LD&, const uint8_t* rec, uint32_t t, uint32_t aux, uint64_t& val) const {
        val = ld_cg_u64(rec + leaf_value_off(t));
        if (aux != l) return false;
        for (uint32_t b = 0; b < l; b++)
            if (rec[b] != byte(b)) return false;
        return true;
    }
};

// Child slot of key byte b among a node's sorted keys (little-endian packed words;
// unused slots repeat the last key), or -1.  The keys are unique, so the slot is the
// position of the FIRST byte equal to b (= the count of keys < b).  Zero-byte test
// on x = word ^ b...b: (x - 0x01..) & ~x & 0x80.. flags every zero byte, and may also
// flag bytes ABOVE a zero byte (borrow) but never below one, so the lowest flag is
// exact.  3 instructions per word instead of the emulated __vcmpltu4/__vcmpeq4 pair.
__device__ __forceinline__ uint32_t zero_bytes(uint32_t w, uint32_t bb) {
    const uint32_t x = w ^ bb;
    return (x - 0x01010101u) & ~x & 0x80808080u;
}
__device__ __forceinline__ int find_key4(uint32_t w0, uint32_t b) {
    const uint32_t z = zero_bytes(w0, b * 0x01010101u);
    return z ? int(__ffs(z) - 1) >> 3 : -1;
}
__device__ __forceinline__ int find_key16(uint32_t w0, uint32_t w1, uint32_t w2, uint32_t w3, uint32_t b) {
    const uint32_t bb = b * 0x01010101u;
    const uint32_t z0 = zero_bytes(w0, bb), z1 = zero_bytes(w1, bb), z2 = zero_bytes(w2, bb), z3 = zero_bytes(w3, bb);
    const uint32_t z = z0 ? z0 : z1 ? z1 : z2 ? z2 : z3;
    const int base = z0 ? 0 : z1 ? 4 : z2 ? 8 : 12;
    return z ? base + (int(__ffs(z) - 1) >> 3) : -1;
}

// Cache policy for the three kinds of dependent loads (B200 L2 is 126 MB; the
// structure of a large index is not).
//   POL 0: plain ld.global.nc everywhere.
//   POL 1: LUT evict_last (keep the root table L2-resident), leaves evict_first.
//   POL 2: as 1 and inner nodes evict_first too.
//   POL 3: LUT evict_last only.
//   POL 4: as 1, plus the L2::64B fetch-size hint on node and leaf loads (a random
//          miss fills 64 B instead of a 128-B line: half the DRAM bytes).
//   POL 5: as 1, L2::64B on leaf loads only.
template <int POL>
struct Loader {
    uint64_t keep, drop, norm;
    static constexpr bool kNode64B = POL == 4;
    static constexpr bool kLeaf64B = POL == 4 || POL == 5;
    static constexpr bool kLeafDrop = POL == 1 || POL == 2 || POL == 4 || POL == 5;
    __device__ __forceinline__ Loader() {
        if (POL != 0) {
            asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(keep));
            asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(drop));
        }
        if (POL == 4) asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(norm));
    }
    template <bool F64 = false>
    __device__ __forceinline__ static uint64_t u64(const void* p, uint64_t pol) {
        uint64_t v;
        if (F64) asm volatile("ld.global.nc.L2::cache_hint.L2::64B.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(pol));
        else asm volatile("ld.global.nc.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(pol));
        return v;
    }
    __device__ __forceinline__ static uint32_t u32(const void* p, uint64_t pol) {
        uint32_t v;
        asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
        return v;
    }
    template <bool F64 = false>
    __device__ __forceinline__ static uint32_t u8(const void* p, uint64_t pol) {
        uint16_t v;
        if (F64) asm volatile("ld.global.nc.L2::cache_hint.L2::64B.u8 %0, [%1], %2;" : "=h"(v) : "l"(p), "l"(pol));
        else asm volatile("ld.global.nc.L2::cache_hint.u8 %0, [%1], %2;" : "=h"(v) : "l"(p), "l"(pol));
        return v;
    }
    template <bool F64 = false>
    __device__ __forceinline__ static uint4 v4(const void* p, uint64_t pol) {
        uint4 v;
        if (F64)
            asm volatile("ld.global.nc.L2::cache_hint.L2::64B.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                         : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p), "l"(pol));
        else
            asm volatile("ld.global.nc.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                         : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p), "l"(pol));
        return v;
    }
    template <bool F64 = false>
    __device__ __forceinline__ static U8x32 v8(const void* p, uint64_t pol) {
        U8x32 v;
        if (F64)
            asm volatile("ld.global.nc.L2::cache_hint.L2::64B.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
                         : "=r"(v.w[0]), "=r"(v.w[1]), "=r"(v.w[2]), "=r"(v.w[3]), "=r"(v.w[4]), "=r"(v.w[5]),
                           "=r"(v.w[6]), "=r"(v.w[7]) : "l"(p), "l"(pol));
        else
            asm volatile("ld.global.nc.L2::cache_hint.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
                         : "=r"(v.w[0]), "=r"(v.w[1]), "=r"(v.w[2]), "=r"(v.w[3]), "=r"(v.w[4]), "=r"(v.w[5]),
                           "=r"(v.w[6]), "=r"(v.w[7]) : "l"(p), "l"(pol));
        return v;
    }
    // LUT entries / blocks
    __device__ __forceinline__ uint64_t lut64(const void* p) const { return POL ? u64(p, keep) : ld_nc_u64(p); }
    __device__ __forceinline__ uint32_t lut32(const void* p) const {
        if (POL) return u32(p, keep);
        uint32_t v;
        asm volatile("ld.global.nc.u32 %0, [%1];" : "=r"(v) : "l"(p));
        return v;
    }
    __device__ __forceinline__ U8x32 lutv8(const void* p) const { return POL ? v8(p, keep) : ld_nc_v8(p); }
    // inner nodes
    __device__ __forceinline__ uint64_t node64(const void* p) const {
        return POL == 2 ? u64(p, drop) : POL == 4 ? u64<true>(p, norm) : ld_nc_u64(p);
    }
    __device__ __forceinline__ uint32_t node8(const void* p) const {
        return POL == 2 ? u8(p, drop) : POL == 4 ? u8<true>(p, norm) : ld_nc_u8(p);
    }
    __device__ __forceinline__ uint4 nodev4(const void* p) const {
        return POL == 2 ? v4(p, drop) : POL == 4 ? v4<true>(p, norm) : ld_nc_v4(p);
    }
    __device__ __forceinline__ U8x32 nodev8(const void* p) const {
        return POL == 2 ? v8(p, drop) : POL == 4 ? v8<true>(p, norm) : ld_nc_v8(p);
    }
    // leaves
    __device__ __forceinline__ uint4 leafv4(const void* p) const {
        return kLeaf64B ? v4<true>(p, drop) : kLeafDrop ? v4(p, drop) : ld_nc_v4(p);
    }
    // Leaf record of a pre-bucketed walk, where a leaf is re-read by the ~8 hit queries
    // of its bucket window: LP 0 = as leafv4 (evict_first + L2::64B), 1 = evict_last +
    // L2::64B, 2 = plain, 3 = evict_last.
    template <int LP>
    __device__ __forceinline__ uint4 leafv4_b(const void* p) const {
        if (LP == 0) return leafv4(p);
        if (LP == 1) return v4<true>(p, keep);
        if (LP == 3) return v4(p, keep);
        return ld_nc_v4(p);
    }
    __device__ __forceinline__ U8x32 leafv8(const void* p) const {   // p 32-B aligned
        return kLeaf64B ? v8<true>(p, drop) : kLeafDrop ? v8(p, drop) : ld_nc_v8(p);
    }
};

// Walk from `link` to a leaf.  Returns the leaf link on a full-key match (its value
// in `val`), 0 otherwise.  With TRACK, `slot` follows the address of the link last
// loaded (the parent's child slot of the leaf found — what a delete unlinks,
// P:137); it starts as the LUT entry address from start_link (0 = root/none).
template <class Key, int POL, bool TRACK = false>
__device__ __forceinline__ uint64_t find_leaf(const DevIndex& ix, const Loader<POL>& ld, const Key& key, uint64_t link,
                                              uint64_t& val, uint64_t* slot = nullptr) {
    const uint32_t len = key.len();
#pragma unroll 1
    for (;;) {
        const uint32_t t = link_type(link);
        const uint64_t idx = link_index(link);
        const uint32_t aux = link_aux(link);
        if (Key::kKind == 4 && t == T_LEAF_HOST) {   // f4: host leaf -> signal (the caller finishes on the host)
            val = idx;
            return link;
        }
        if (t >= T_LEAF8) {
            const uint8_t* rec = ix.base[t] + idx * record_bytes(t);
            return key.leaf_match(ld, rec, t, aux, val) ? link : 0;
        }
        if (t == T_NULL || aux >= len) return 0;
        const uint32_t b = key.byte(aux);
        const uint8_t* rec = ix.base[t] + idx * record_bytes(t);
        if (t == T_N256) {
            link = ld.node64(rec + kN256Child + 8 * b);
            if (TRACK) *slot = uint64_t(rec + kN256Child + 8 * b);
        } else if (t == T_N48) {
            const uint32_t s = ld.node8(rec + kN48Index + b);
            if (s == kN48Empty) return 0;
            link = ld.node64(rec + kN48Child + 8 * s);
            if (TRACK) *slot = uint64_t(rec + kN48Child + 8 * s);
        } else if (t == T_N16) {
            const uint4 k4 = ld.nodev4(rec + kN16Keys);
            const int c = find_key16(k4.x, k4.y, k4.z, k4.w, b);
            if (c < 0) return 0;
            link = ld.node64(rec + kN16Child + 8 * c);
            if (TRACK) *slot = uint64_t(rec + kN16Child + 8 * c);
        } else {  // N4: keys + child[0..2] in one 256-bit load; child[3] (same line) if taken
            const U8x32 r = ld.nodev8(rec);
            const int c = find_key4(r.w[0], b);
            if (c < 0) return 0;
            const uint32_t less = uint32_t(c);
            if (less == 3) {
                link = ld.node64(rec + kN4Child + 24);
            } else {
                const uint32_t lo = less == 0 ? r.w[2] : less == 1 ? r.w[4] : r.w[6];
                const uint32_t hi = less == 0 ? r.w[3] : less == 1 ? r.w[5] : r.w[7];
                link = uint64_t(lo) | (uint64_t(hi) << 32);
            }
            if (TRACK) *slot = uint64_t(rec + kN4Child + 8 * less);
        }
    }
}

// Compact 32-bit LUT entry (integer keys only; layout.h): [31:29] type; leaves
// [28:0] index; inner nodes [28:26] branch depth - k, [25:0] index.
__device__ __forceinline__ uint64_t expand_lut32(uint32_t e, uint32_t k, uint32_t leaf_len) {
    const uint32_t t = e >> 29;
    if (t == T_NULL) return 0;
    if (t >= T_LEAF8) return make_link(t, leaf_len, e & 0x1FFFFFFFu);
    return make_link(t, k + ((e >> 26) & 7u), e & 0x3FFFFFFu);
}

// Rank-form LUT entry p (capi.cu rank_lut): one 256-bit read of a 32-B block per
// 32 entries (the whole table is 1 B/entry and stays L2-resident).  Type from three
// bit-planes, index = per-type base + popcount of earlier same-type entries;
// exceptions (leaves, other depths, non-consecutive indices) go to the link table.
template <int POL, bool TRACK = false>
__device__ __forceinline__ uint64_t decode_lut_rank(const DevIndex& ix, const Loader<POL>& ld, const U8x32& blk,
                                                    uint64_t p, uint64_t* slot = nullptr) {
    const uint32_t j = uint32_t(p & 31);
    if ((blk.w[3] >> j) & 1) {
        if (TRACK) *slot = uint64_t(ix.lut + p);
        return ld.lut64(ix.lut + p);
    }
    const uint32_t p0 = blk.w[0], p1 = blk.w[1], p2 = blk.w[2];
    const uint32_t t = ((p0 >> j) & 1) | (((p1 >> j) & 1) << 1) | (((p2 >> j) & 1) << 2);
    if (t == T_NULL) return 0;
    const uint32_t m = ((t & 1) ? p0 : ~p0) & ((t & 2) ? p1 : ~p1) & ((t & 4) ? p2 : ~p2) & ((1u << j) - 1);
    const uint32_t base = t == T_N4 ? blk.w[4] : t == T_N16 ? blk.w[5] : t == T_N48 ? blk.w[6] : blk.w[7];
    return make_link(t, ix.lut_bytes, uint64_t(base) + __popc(m));
}
template <int POL, bool TRACK = false>
__device__ __forceinline__ uint64_t expand_lut_rank(const DevIndex& ix, const Loader<POL>& ld, uint64_t p,
                                                    uint64_t* slot = nullptr) {
    return decode_lut_rank<POL, TRACK>(ix, ld, ld.lutv8(ix.lutr + (p >> 5) * 2), p, slot);
}

// Start of a walk: LUT[first k key bytes] or the root.  With TRACK, *slot =
// address of the LUT entry holding the link (bit 0 set for a 32-bit entry), 0 if
// the start is the root (a root leaf is never unlinked; its tombstone suffices).
// Wide root table ("merged top layers", B200 reading): entry p is 32 B =
// {link, the 4 / 16 sorted key bytes of the N4 / N16 it points to, leaf run or 0}.  One
// 32-B request brings the start link AND the first node's search keys, so the walk
// skips that node's key read and loads the child link directly: on c3 one L2
// request less for every query whose LUT target is an N16, a 32-B request
// replaced by an 8-B one for N4 targets.  Deletes never change a node's keys (they
// null child links, reading C18), so the embedded keys stay a superset filter.
template <class Key, int POL>
__device__ __forceinline__ uint64_t decode_wide(const DevIndex& ix, const Loader<POL>& ld, const Key& key, const U8x32& e) {
    const uint64_t link = uint64_t(e.w[0]) | (uint64_t(e.w[1]) << 32);
    const uint32_t t = link_type(link);
    const uint64_t run = uint64_t(e.w[6]) | (uint64_t(e.w[7]) << 32);
    const uint32_t aux = link_aux(link);
    if (t == T_N256 && run)                                    // full N256 of leaves: child b = run + b
        return aux >= key.len() ? 0 : run + key.byte(aux);
    if (t != T_N4 && t != T_N16) return link;
    if (aux >= key.len()) return 0;
    // The entry's 16 key bytes are the N16's keys, or the N4's padded with its last
    // key (capi.cu), so both take the same branch-free search.
    const int c = find_key16(e.w[2], e.w[3], e.w[4], e.w[5], key.byte(aux));
    if (c < 0) return 0;
    // Leaf run (layout.h leaf_run_link): when every child of the node is a leaf, the
    // leaves are consecutive in the lexicographically ordered leaf buffer,
    // so child c's link is run + c and the child-link request disappears too.  A
    // child nulled by a delete (C18) leaves a tombstoned leaf (value CUART_MISS)
    // at run + c, which every caller already reads as absent.
    if (run) return run + c;
    const uint8_t* rec = ix.base[t] + link_index(link) * record_bytes(t);
    return ld.node64(rec + (t == T_N4 ? kN4Child : kN16Child) + 8 * c);
}
template <class Key, int POL>
__device__ __forceinline__ uint64_t start_wide(const DevIndex& ix, const Loader<POL>& ld, const Key& key, uint64_t p) {
    return decode_wide(ix, ld, key, ld.lutv8(ix.lutw + p * 4));
}

// Skip table ("merged upper layers", for byte strings whose first bytes do
// not discriminate: c4's keys share 6-byte segments, so the 3-byte root table skips
// one level only).  Entry = the node covering every key with a given D-byte prefix
// (the first node on the path whose branch depth is >= D, or the leaf), so a walk
// can start there; a prefix absent from the table belongs to no key of length >= D.
// One 32-B request (the table is small and L2-resident) replaces the top levels.
template <int POL>
__device__ __forceinline__ uint64_t skip_start(const DevIndex& ix, const Loader<POL>& ld, const KeyBytes& key) {
    const uint32_t D = ix.skip_d;
    const uint64_t p0 = key.w[0] & low_bytes_mask(D < 8 ? D : 8u);
    const uint64_t p1 = D > 8 ? key.w[1] & low_bytes_mask(D - 8) : 0ull;
    uint64_t h = skip_hash(p0, p1) & ix.skip_mask;
#pragma unroll 1
    for (;;) {
        const U8x32 e = ld.lutv8(ix.skip + 4 * h);
        const uint64_t link = uint64_t(e.w[4]) | (uint64_t(e.w[5]) << 32);
        if (link == 0) return 0;
        if ((uint64_t(e.w[0]) | (uint64_t(e.w[1]) << 32)) == p0 && (uint64_t(e.w[2]) | (uint64_t(e.w[3]) << 32)) == p1)
            return link;
        h = (h + 1) & ix.skip_mask;
    }
}

template <class Key, int POL, bool TRACK = false>
__device__ __forceinline__ uint64_t start_link(const DevIndex& ix, const Loader<POL>& ld, const Key& key,
                                               uint64_t* slot = nullptr) {
    if constexpr (Key::kKind == 3 && !TRACK) {
        if (ix.skip && key.len() >= ix.skip_d) return skip_start(ix, ld, key);
    }
    if (TRACK) *slot = 0;
    if (ix.lut_bytes && key.len() >= ix.lut_bytes) {
        const uint64_t p = key.prefix(ix.lut_bytes);
        if (!TRACK && ix.walk_wide) return start_wide(ix, ld, key, p);
        if (ix.lutr) return expand_lut_rank<POL, TRACK>(ix, ld, p, slot);
        if (ix.lut32) {
            if (TRACK) *slot = uint64_t(ix.lut32 + p) | 1u;
            return expand_lut32(ld.lut32(ix.lut32 + p), ix.lut_bytes, ix.fixed_len);
        }
        if (TRACK) *slot = uint64_t(ix.lut + p);
        return ld.lut64(ix.lut + p);
    }
    return ix.root;
}

}  // namespace cuart
