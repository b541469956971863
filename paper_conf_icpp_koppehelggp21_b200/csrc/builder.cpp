// builder.cpp — host-side canonical ART build and flattening (§4.1
// P:153-155 "Populating the ART index" / "Mapping the CPU ART into the buffer
// structure described in chapter 3.2.1").
//
// B200 reading: instead of inserting keys one by one into a pointer ART and then
// walking it (the paper's populate -> map), the builder bulk-loads the same
// canonical tree straight from the sorted key set: an insert-only,
// path-compressed, lazily-expanded ART [17] over a prefix-free key set is a
// function of the key set alone, with one inner node per maximal group of >= 2
// keys sharing a prefix, branching at the group's first differing byte.  Groups
// are processed level by level (breadth first, OpenMP-parallel inside a level),
// which numbers the inner nodes of every type in BFS order (reading C10) and
// leaves in lexicographic order per leaf class.
#include <string.h>

#include <algorithm>
#include <parallel/algorithm>
#include <vector>

#include <omp.h>

#include "../../include/cuart.h"
#include "builder.h"

namespace cuart {
namespace {

struct SortedKeys {
    uint32_t fixed_len = 0;             // 4 / 8 for integer kinds, 0 for byte strings
    bool is_long = false;               // CUART_KEY_LONG: variable-length keys in lbytes / loff
    std::vector<uint64_t> ik;           // integer kinds: numeric key (big-endian byte order = numeric order)
    std::vector<uint8_t> slots;         // byte strings: n x 32 zero-padded
    std::vector<uint8_t> lens;
    std::vector<uint8_t> lbytes;        // long keys: concatenated, sorted
    std::vector<uint64_t> loff;         // long keys: [n + 1]
    std::vector<uint64_t> vals;
    uint64_t n = 0;

    inline const uint8_t* kptr(uint64_t i) const { return is_long ? &lbytes[loff[i]] : &slots[i * kMaxKey]; }
    inline uint32_t byte(uint64_t i, uint32_t d) const {
        if (fixed_len) return uint32_t(ik[i] >> (8 * (fixed_len - 1 - d))) & 0xFF;
        return kptr(i)[d];
    }
    inline uint32_t len(uint64_t i) const {
        return fixed_len ? fixed_len : is_long ? uint32_t(loff[i + 1] - loff[i]) : lens[i];
    }
    // Equal bytes of keys i and j from byte `from` on, bounded by the shorter key.
    inline uint32_t lcp(uint64_t i, uint64_t j, uint32_t from) const {
        if (fixed_len) {
            uint64_t x = ik[i] ^ ik[j];
            uint32_t total = x ? uint32_t(__builtin_clzll(x) - (64 - 8 * fixed_len)) / 8 : fixed_len;
            return total - from;
        }
        uint32_t m = std::min(len(i), len(j));
        const uint8_t* a = kptr(i);
        const uint8_t* b = kptr(j);
        uint32_t p = from;
        while (p < m && a[p] == b[p]) p++;
        return p - from;
    }
    inline void write_key(uint64_t i, uint8_t* dst) const {   // canonical bytes, zero padded by caller
        if (fixed_len) {
            for (uint32_t b = 0; b < fixed_len; b++) dst[b] = uint8_t(ik[i] >> (8 * (fixed_len - 1 - b)));
        } else {
            memcpy(dst, kptr(i), len(i));
        }
    }
    inline uint64_t prefix_k(uint64_t i, uint32_t k) const {
        uint64_t p = 0;
        for (uint32_t b = 0; b < k; b++) p = (p << 8) | byte(i, b);
        return p;
    }
};

struct StrRec {
    uint64_t w[4];
    uint32_t len;
    uint32_t pad;
    uint64_t idx;
};

inline uint64_t load_be64(const uint8_t* p) {
    uint64_t v = 0;
    for (int b = 0; b < 8; b++) v = (v << 8) | p[b];
    return v;
}

// f4: variable-length keys (1..255 B): sort the key indices lexicographically
// (shorter first on a common prefix), keep the LAST occurrence of a duplicate
// (reading C6), check prefix-freeness (reading C3).
int canonicalize_long(const uint8_t* data, const uint64_t* off, const uint64_t* values, uint64_t n, SortedKeys& S) {
    for (uint64_t i = 0; i < n; i++) {
        if (off[i + 1] < off[i]) return CUART_ERR_INVALID_ARGUMENT;
        const uint64_t l = off[i + 1] - off[i];
        if (l == 0 || l > kMaxLongKey) return CUART_ERR_KEY_LENGTH;
    }
    std::vector<uint64_t> ord(n);
    for (uint64_t i = 0; i < n; i++) ord[i] = i;
    auto cmp3 = [&](uint64_t a, uint64_t b) {
        const uint64_t la = off[a + 1] - off[a], lb = off[b + 1] - off[b];
        const int c = memcmp(data + off[a], data + off[b], std::min(la, lb));
        return c != 0 ? c : (la < lb ? -1 : la > lb ? 1 : 0);
    };
    __gnu_parallel::sort(ord.begin(), ord.end(), [&](uint64_t a, uint64_t b) {
        const int c = cmp3(a, b);
        return c != 0 ? c < 0 : a < b;
    });
    S.is_long = true;
    S.loff.push_back(0);
    for (uint64_t i = 0; i < n; i++) {
        if (i + 1 < n && cmp3(ord[i], ord[i + 1]) == 0) continue;
        const uint64_t k = ord[i], l = off[k + 1] - off[k];
        S.lbytes.insert(S.lbytes.end(), data + off[k], data + off[k] + l);
        S.loff.push_back(S.lbytes.size());
        S.vals.push_back(values[k]);
    }
    S.n = S.vals.size();
    for (uint64_t j = 0; j + 1 < S.n; j++)
        if (S.len(j) < S.len(j + 1) && S.lcp(j, j + 1, 0) >= S.len(j)) return CUART_ERR_NOT_PREFIX_FREE;
    return CUART_OK;
}

int canonicalize(uint32_t kind, const void* data, const uint8_t* lengths, const uint64_t* values, uint64_t n,
                 SortedKeys& S, const uint64_t* long_offsets) {
    for (uint64_t i = 0; i < n; i++)
        if (values[i] == kMiss) return CUART_ERR_RESERVED_VALUE;
    if (kind == CUART_KEY_LONG) {
        if (!long_offsets) return CUART_ERR_INVALID_ARGUMENT;
        return canonicalize_long((const uint8_t*)data, long_offsets, values, n, S);
    }
    if (kind == CUART_KEY_U64 || kind == CUART_KEY_U32) {
        S.fixed_len = kind == CUART_KEY_U64 ? 8 : 4;
        std::vector<std::pair<uint64_t, uint64_t>> kv(n);
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < int64_t(n); i++)
            kv[i] = {kind == CUART_KEY_U64 ? ((const uint64_t*)data)[i] : uint64_t(((const uint32_t*)data)[i]),
                     uint64_t(i)};
        __gnu_parallel::sort(kv.begin(), kv.end());
        // dedupe: keep the LAST occurrence of each key (reading C6: last wins)
        S.ik.reserve(n);
        S.vals.reserve(n);
        for (uint64_t i = 0; i < n; i++) {
            if (i + 1 < n && kv[i + 1].first == kv[i].first) continue;
            S.ik.push_back(kv[i].first);
            S.vals.push_back(values[kv[i].second]);
        }
        S.n = S.ik.size();
        return CUART_OK;
    }
    if (kind != CUART_KEY_BYTES || lengths == nullptr) return CUART_ERR_INVALID_ARGUMENT;
    const uint8_t* slots = (const uint8_t*)data;
    for (uint64_t i = 0; i < n; i++)
        if (lengths[i] == 0 || lengths[i] > kMaxKey) return CUART_ERR_KEY_LENGTH;
    std::vector<StrRec> recs(n);
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < int64_t(n); i++) {
        uint8_t tmp[kMaxKey] = {0};
        memcpy(tmp, slots + i * kMaxKey, lengths[i]);   // bytes past the length are ignored
        for (int w = 0; w < 4; w++) recs[i].w[w] = load_be64(tmp + 8 * w);
        recs[i].len = lengths[i];
        recs[i].pad = 0;
        recs[i].idx = uint64_t(i);
    }
    __gnu_parallel::sort(recs.begin(), recs.end(), [](const StrRec& a, const StrRec& b) {
        for (int w = 0; w < 4; w++)
            if (a.w[w] != b.w[w]) return a.w[w] < b.w[w];
        if (a.len != b.len) return a.len < b.len;
        return a.idx < b.idx;
    });
    auto same = [](const StrRec& a, const StrRec& b) {
        return a.len == b.len && a.w[0] == b.w[0] && a.w[1] == b.w[1] && a.w[2] == b.w[2] && a.w[3] == b.w[3];
    };
    std::vector<uint64_t> keep;
    keep.reserve(n);
    for (uint64_t i = 0; i < n; i++) {
        if (i + 1 < n && same(recs[i + 1], recs[i])) continue;
        keep.push_back(i);
    }
    S.n = keep.size();
    S.slots.assign(S.n * kMaxKey, 0);
    S.lens.resize(S.n);
    S.vals.resize(S.n);
#pragma omp parallel for schedule(static)
    for (int64_t j = 0; j < int64_t(S.n); j++) {
        const StrRec& r = recs[keep[j]];
        uint8_t* dst = &S.slots[j * kMaxKey];
        for (int w = 0; w < 4; w++)
            for (int b = 0; b < 8; b++) dst[8 * w + b] = uint8_t(r.w[w] >> (8 * (7 - b)));
        S.lens[j] = uint8_t(r.len);
        S.vals[j] = values[r.idx];
    }
    // prefix-freeness: in lexicographic order a key that is a proper prefix of
    // another is a proper prefix of its successor.
    for (uint64_t j = 0; j + 1 < S.n; j++)
        if (S.lens[j] < S.lens[j + 1] && S.lcp(j, j + 1, 0) >= S.lens[j]) return CUART_ERR_NOT_PREFIX_FREE;
    return CUART_OK;
}

struct Group {
    uint64_t lo, hi;         // key range [lo, hi), >= 2 keys
    uint32_t depth;          // first key byte not yet consumed
    int32_t pdepth;          // parent's branch depth (-1 for the root)
    uint32_t ptype;          // parent's type (0 = this is the root)
    uint32_t pslot;          // child slot in the parent record
    uint64_t pidx;           // parent's index in its type buffer
};

inline uint32_t type_for_count(uint32_t c) { return c <= 4 ? T_N4 : c <= 16 ? T_N16 : c <= 48 ? T_N48 : T_N256; }

inline uint64_t* child_slot(HostLayout& L, uint32_t type, uint64_t idx, uint32_t slot) {
    uint8_t* rec = L.buf[type].data() + idx * kRecordBytes[type];
    switch (type) {
    case T_N4: return (uint64_t*)(rec + kN4Child) + slot;
    case T_N16: return (uint64_t*)(rec + kN16Child) + slot;
    case T_N48: return (uint64_t*)(rec + kN48Child) + slot;
    default: return (uint64_t*)(rec + kN256Child) + slot;
    }
}

}  // namespace

int build_host_layout(uint32_t kind, const void* data, const uint8_t* lengths, const uint64_t* values, uint64_t n,
                      uint32_t lut_bytes, HostLayout& L, const uint64_t* long_offsets) {
    if (kind < CUART_KEY_U32 || kind > CUART_KEY_LONG) return CUART_ERR_INVALID_ARGUMENT;
    if (lut_bytes > 3) return CUART_ERR_INVALID_ARGUMENT;
    if (n > 0 && (data == nullptr || values == nullptr)) return CUART_ERR_INVALID_ARGUMENT;
    L = HostLayout();
    L.key_kind = kind;
    L.lut_bytes = lut_bytes;
    SortedKeys S;
    if (n > 0) {
        int rc = canonicalize(kind, data, lengths, values, n, S, long_offsets);
        if (rc != CUART_OK) return rc;
    }
    L.n_keys = S.n;
    if (lut_bytes) L.lut.assign(uint64_t(1) << (8 * lut_bytes), 0);
    const uint32_t K = lut_bytes;

    // leaf class ranks: leaves are numbered in lexicographic order per class
    auto leaf_type = [](uint32_t len) { return len > kMaxKey ? uint32_t(T_LEAF_HOST) : leaf_type_for_len(len); };
    std::vector<uint64_t> leaf_rank(S.n);
    {
        uint64_t c[9] = {0};
        for (uint64_t i = 0; i < S.n; i++) leaf_rank[i] = c[leaf_type(S.len(i))]++;
        for (uint32_t t = T_LEAF8; t <= T_LEAF32; t++) {
            L.count[t] = c[t];
            if (c[t] > kIndexMask) return CUART_ERR_TOO_LARGE;
            L.buf[t].assign(c[t] * kRecordBytes[t], 0);
            if (kind == CUART_KEY_BYTES) L.leaf_len[t].assign(c[t], 0);
        }
        if (kind == CUART_KEY_BYTES)
            for (uint64_t i = 0; i < S.n; i++) L.leaf_len[leaf_type(S.len(i))][leaf_rank[i]] = uint8_t(S.len(i));
        // f4: host-resident long leaves, in lexicographic order like every leaf class
        L.long_off.assign(1, 0);
        for (uint64_t i = 0; i < S.n; i++) {
            if (leaf_type(S.len(i)) != T_LEAF_HOST) continue;
            L.long_bytes.insert(L.long_bytes.end(), S.kptr(i), S.kptr(i) + S.len(i));
            L.long_off.push_back(L.long_bytes.size());
            L.long_vals.push_back(S.vals[i]);
        }
    }
    auto write_leaf = [&](uint64_t i) -> uint64_t {
        uint32_t len = S.len(i);
        uint32_t t = leaf_type(len);
        if (t == T_LEAF_HOST) return make_link(t, len, leaf_rank[i]);
        uint8_t* rec = L.buf[t].data() + leaf_rank[i] * kRecordBytes[t];
        S.write_key(i, rec);
        memcpy(rec + kLeafValueOff[t], &S.vals[i], 8);
        return make_link(t, len, leaf_rank[i]);
    };

    if (S.n == 0) { L.root = 0; return CUART_OK; }
    if (S.n == 1) {
        L.root = write_leaf(0);
        L.max_depth = 1;
        if (K && S.len(0) >= K) L.lut[S.prefix_k(0, K)] = L.root;
        return CUART_OK;
    }

    std::vector<Group> cur{Group{0, S.n, 0, -1, 0, 0, 0}}, next;
    uint32_t level = 0;
    while (!cur.empty()) {
        level++;
        const int64_t G = int64_t(cur.size());
        std::vector<uint32_t> bd(G), cnt(G), multi(G);
        // pass 1: branch depth, child count, number of multi-key children
#pragma omp parallel for schedule(dynamic, 256)
        for (int64_t g = 0; g < G; g++) {
            const Group& gr = cur[g];
            uint32_t p = S.lcp(gr.lo, gr.hi - 1, gr.depth);      // sorted: lcp(first,last) = group lcp
            uint32_t d = gr.depth + p;
            uint32_t c = 0, m = 0;
            uint64_t a = gr.lo;
            while (a < gr.hi) {
                uint32_t b = S.byte(a, d);                         // prefix-free: every key has byte d
                uint64_t e = a + 1;
                while (e < gr.hi && S.byte(e, d) == b) e++;
                c++;
                if (e - a > 1) m++;
                a = e;
            }
            bd[g] = d;
            cnt[g] = c;
            multi[g] = m;
        }
        // pass 2: BFS numbering per type, next-level offsets
        std::vector<uint64_t> nidx(G), noff(G);
        uint64_t tcount[5] = {L.count[0], L.count[1], L.count[2], L.count[3], L.count[4]};
        uint64_t nnext = 0;
        for (int64_t g = 0; g < G; g++) {
            uint32_t t = type_for_count(cnt[g]);
            nidx[g] = tcount[t]++;
            noff[g] = nnext;
            nnext += multi[g];
        }
        for (uint32_t t = T_N4; t <= T_N256; t++) {
            if (tcount[t] > kIndexMask) return CUART_ERR_TOO_LARGE;
            if (tcount[t] != L.count[t]) L.buf[t].resize(tcount[t] * kRecordBytes[t], 0);
            L.count[t] = tcount[t];
        }
        next.assign(nnext, Group{});
        // pass 3: write records, leaves, parent links, LUT entries
#pragma omp parallel for schedule(dynamic, 256)
        for (int64_t g = 0; g < G; g++) {
            const Group& gr = cur[g];
            const uint32_t d = bd[g], c = cnt[g], t = type_for_count(c);
            const uint64_t idx = nidx[g];
            const uint64_t link = make_link(t, d, idx);
            if (gr.ptype == 0) L.root = link;
            else *child_slot(L, gr.ptype, gr.pidx, gr.pslot) = link;
            if (K && gr.pdepth < int32_t(K) && d >= K) L.lut[S.prefix_k(gr.lo, K)] = link;

            uint8_t* rec = L.buf[t].data() + idx * kRecordBytes[t];
            uint8_t* hdr = rec + header_off(t);
            const uint32_t plen = d - gr.depth;
            hdr[0] = uint8_t(plen);
            hdr[1] = uint8_t(c - 1);
            for (uint32_t b = 0; b < plen && b < kHeaderPrefix; b++) hdr[2 + b] = uint8_t(S.byte(gr.lo, gr.depth + b));
            if (t == T_N48) memset(rec + kN48Index, kN48Empty, 256);
            uint64_t a = gr.lo, off = noff[g];
            uint32_t j = 0, lastb = 0;
            while (a < gr.hi) {
                uint32_t b = S.byte(a, d);
                uint64_t e = a + 1;
                while (e < gr.hi && S.byte(e, d) == b) e++;
                uint32_t slot = (t == T_N256) ? b : j;
                if (t == T_N4) rec[kN4Keys + j] = uint8_t(b);
                else if (t == T_N16) rec[kN16Keys + j] = uint8_t(b);
                else if (t == T_N48) rec[kN48Index + b] = uint8_t(j);
                if (e - a == 1) {
                    uint64_t ll = write_leaf(a);
                    *child_slot(L, t, idx, slot) = ll;
                    if (K && d < K && S.len(a) >= K) L.lut[S.prefix_k(a, K)] = ll;
                } else {
                    next[off++] = Group{a, e, d + 1, int32_t(d), t, slot, idx};
                }
                lastb = b;
                j++;
                a = e;
            }
            // unused N4/N16 key slots repeat the last key (layout.h)
            if (t == T_N4) for (uint32_t q = j; q < 4; q++) rec[kN4Keys + q] = uint8_t(lastb);
            if (t == T_N16) for (uint32_t q = j; q < 16; q++) rec[kN16Keys + q] = uint8_t(lastb);
        }
        cur.swap(next);
        next.clear();
    }
    L.max_depth = level + 1;
    return CUART_OK;
}

// ---------------------------------------------------------------------------------------------
// CPU lookup engine over the flat layout (§4.2 Fig. 7).  Same traversal as the GPU
// kernel: optimistic prefix skip via the branch depth in the link, full-key compare at the leaf.
namespace {

struct QView {
    uint32_t kind;
    const void* data;
    const uint8_t* lens;
    inline uint32_t len(uint64_t i) const { return kind == CUART_KEY_U64 ? 8 : kind == CUART_KEY_U32 ? 4 : lens[i]; }
    inline void bytes(uint64_t i, uint8_t* out32) const {
        memset(out32, 0, kMaxKey);
        if (kind == CUART_KEY_U64) {
            uint64_t k = ((const uint64_t*)data)[i];
            for (int b = 0; b < 8; b++) out32[b] = uint8_t(k >> (8 * (7 - b)));
        } else if (kind == CUART_KEY_U32) {
            uint32_t k = ((const uint32_t*)data)[i];
            for (int b = 0; b < 4; b++) out32[b] = uint8_t(k >> (8 * (3 - b)));
        } else {
            uint32_t l = lens[i] > kMaxKey ? kMaxKey : lens[i];
            memcpy(out32, (const uint8_t*)data + i * kMaxKey, l);
        }
    }
};

// Number of distinct 32-byte sectors covered by [off, off+bytes) of a buffer whose
// base is 256-byte aligned in the device arena (so record offsets decide).
inline uint32_t sectors(uint64_t off, uint32_t bytes) { return uint32_t((off + bytes - 1) / 32 - off / 32 + 1); }

// Walk one key.  If `sec` is non-null, add the 32-byte sectors the GPU kernel
// (kernels.cuh find_leaf) reads on this path: LUT entry 8 B; N256 child 8 B;
// N48 index byte + child 8 B; N16 keys 16 B + child 8 B; N4 bytes [16, 56) of its
// 64-B record; leaves 16 / 32 / 48 B.
// wide: the walk starts from the 32-B wide root-table entry (link + the target
// N4/N16's keys, kernels.cuh start_wide) and reads that node's child link directly.
uint64_t walk_one(const HostLayout& L, const uint8_t* key, uint32_t len, uint32_t* sec = nullptr, bool wide = false,
                  uint32_t skip_d = 0) {
    if (len == 0 || len > kMaxKey) return kMiss;
    uint32_t s = 0;
    uint64_t link = L.root;
    struct Guard { uint32_t* dst; uint32_t* s; ~Guard() { if (dst) *dst = *s; } } guard{sec, &s};
    if (skip_d && len >= skip_d && L.key_kind == CUART_KEY_BYTES) {
        // the device's skip table (capi.cu build_skip_table): one 32-B probe yields the
        // node covering the query's first skip_d bytes; the levels above it are not read
        s += 1;
        if (L.lut_bytes && skip_d >= L.lut_bytes) {
            uint64_t p = 0;
            for (uint32_t b = 0; b < L.lut_bytes; b++) p = (p << 8) | key[b];
            link = L.lut[p];
        }
        for (;;) {
            const uint32_t t = link_type(link);
            if (t == T_NULL) return kMiss;
            if (t >= T_LEAF8 || link_aux(link) >= skip_d) break;
            const uint8_t* rec = L.buf[t].data() + link_index(link) * kRecordBytes[t];
            const uint8_t b = key[link_aux(link)];
            uint64_t child = 0;
            if (t == T_N256) memcpy(&child, rec + kN256Child + 8 * b, 8);
            else if (t == T_N48) {
                if (rec[kN48Index + b] == kN48Empty) return kMiss;
                memcpy(&child, rec + kN48Child + 8 * rec[kN48Index + b], 8);
            } else {
                const uint8_t* keys = rec + (t == T_N4 ? kN4Keys : kN16Keys);
                const uint32_t nk = t == T_N4 ? 4 : 16;
                uint32_t c = nk;
                for (uint32_t j = 0; j < nk; j++)
                    if (keys[j] == b) {
                        c = j;
                        break;
                    }
                if (c == nk) return kMiss;
                memcpy(&child, rec + (t == T_N4 ? kN4Child : kN16Child) + 8 * c, 8);
            }
            link = child;
        }
    } else if (L.lut_bytes && len >= L.lut_bytes) {
        uint64_t p = 0;
        for (uint32_t b = 0; b < L.lut_bytes; b++) p = (p << 8) | key[b];
        link = L.lut[p];
        s += sectors(p * (wide ? 32 : 8), wide ? 32 : 8);
        const uint32_t t = link_type(link);
        if (wide && t == T_N256 && link_aux(link) < len &&
            leaf_run_link(L.buf[t].data() + link_index(link) * kRecordBytes[t], t)) {   // full N256 of leaves
            memcpy(&link, L.buf[t].data() + link_index(link) * kRecordBytes[t] + kN256Child + 8 * key[link_aux(link)], 8);
        } else if (wide && (t == T_N4 || t == T_N16)) {
            const uint32_t d = link_aux(link);
            if (d >= len) return kMiss;
            const uint64_t roff = link_index(link) * kRecordBytes[t];
            const uint8_t* rec = L.buf[t].data() + roff;
            const uint32_t nk = t == T_N4 ? 4 : 16;
            const uint8_t* keys = rec + (t == T_N4 ? kN4Keys : kN16Keys);
            uint32_t less = 0, eq = 0;
            for (uint32_t j = 0; j < nk; j++) { less += keys[j] < key[d]; eq |= keys[j] == key[d]; }
            if (!eq) return kMiss;
            const uint64_t co = roff + (t == T_N4 ? kN4Child : kN16Child) + 8 * less;
            const uint64_t run = leaf_run_link(rec, t);   // leaf run: no child-link read
            if (!run) s += sectors(co, 8);
            memcpy(&link, L.buf[t].data() + co, 8);
        }
    }
    for (;;) {
        const uint32_t t = link_type(link);
        if (t == T_NULL) return kMiss;
        const uint64_t idx = link_index(link);
        const uint64_t roff = idx * kRecordBytes[t];
        const uint8_t* rec = L.buf[t].data() + roff;
        if (t >= T_LEAF8) {
            s += sectors(roff, kRecordBytes[t]);
            if (link_aux(link) != len) return kMiss;
            if (memcmp(rec, key, kLeafKeyBytes[t]) != 0) return kMiss;
            uint64_t v;
            memcpy(&v, rec + kLeafValueOff[t], 8);
            return v;
        }
        const uint32_t d = link_aux(link);
        if (d >= len) return kMiss;
        const uint8_t b = key[d];
        if (t == T_N256) {
            s += sectors(roff + kN256Child + 8 * b, 8);
            memcpy(&link, rec + kN256Child + 8 * b, 8);
        } else if (t == T_N48) {
            s += sectors(roff + kN48Index + b, 1);
            uint8_t slot = rec[kN48Index + b];
            if (slot == kN48Empty) return kMiss;
            s += sectors(roff + kN48Child + 8 * slot, 8);
            memcpy(&link, rec + kN48Child + 8 * slot, 8);
        } else {
            const uint32_t nk = t == T_N4 ? 4 : 16;
            const uint8_t* keys = rec + (t == T_N4 ? kN4Keys : kN16Keys);
            s += t == T_N4 ? sectors(roff, 32) : sectors(roff + kN16Keys, 16);
            uint32_t less = 0, eq = 0;
            for (uint32_t j = 0; j < nk; j++) { less += keys[j] < b; eq |= keys[j] == b; }
            if (!eq) return kMiss;
            if (t == T_N16) s += sectors(roff + kN16Child + 8 * less, 8);
            if (t == T_N4 && less == 3) s += sectors(roff + kN4Child + 24, 8);
            memcpy(&link, rec + (t == T_N4 ? kN4Child : kN16Child) + 8 * less, 8);
        }
    }
}

}  // namespace

void host_layout_sectors(const HostLayout& L, uint32_t kind, const void* queries, const uint8_t* lengths, uint64_t n,
                         uint32_t* sec, int threads, bool wide, uint32_t skip_d) {
    QView q{kind, queries, lengths};
    if (threads <= 0) threads = omp_get_max_threads();
#pragma omp parallel for schedule(static) num_threads(threads)
    for (int64_t i = 0; i < int64_t(n); i++) {
        uint8_t key[kMaxKey];
        q.bytes(i, key);
        sec[i] = 0;
        walk_one(L, key, q.len(i), &sec[i], wide, skip_d);
    }
}

void host_layout_lookup(const HostLayout& L, uint32_t kind, const void* queries, const uint8_t* lengths, uint64_t n,
                        uint64_t* out, int threads) {
    QView q{kind, queries, lengths};
    if (threads <= 0) threads = omp_get_max_threads();
#pragma omp parallel for schedule(static) num_threads(threads)
    for (int64_t i = 0; i < int64_t(n); i++) {
        uint8_t key[kMaxKey];
        q.bytes(i, key);
        out[i] = walk_one(L, key, q.len(i));
    }
}

}  // namespace cuart
