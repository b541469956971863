// builder.h — host-side canonical ART build + flattening into the CuART layout.
#pragma once
#include <stdint.h>

#include <vector>

#include "layout.h"

namespace cuart {

struct HostLayout {
    uint32_t key_kind = 0;                 // cuart_key_kind
    std::vector<uint8_t> buf[8];           // raw records per type code (1..7)
    uint64_t count[8] = {0};
    uint64_t root = 0;                     // packed root link (0 = empty tree)
    uint32_t lut_bytes = 0;
    std::vector<uint64_t> lut;             // 2^(8*lut_bytes) links, or empty
    uint64_t n_keys = 0;
    uint32_t max_depth = 0;
    // f4 (CUART_KEY_LONG): host-resident leaves of keys longer than kMaxKey (P:126
    // option 2), in lexicographic order; link T_LEAF_HOST, index = position here.
    std::vector<uint8_t> long_bytes;       // concatenated keys
    std::vector<uint64_t> long_off;        // [count + 1] offsets into long_bytes
    std::vector<uint64_t> long_vals;
    // BYTES: key length of every leaf, per leaf class in leaf order (range queries,
    // the order of two keys whose zero-padded bytes agree is decided by length)
    std::vector<uint8_t> leaf_len[8];
};

// Status codes mirror cuart_status (include/cuart.h).
// kind CUART_KEY_LONG: data = concatenated key bytes, `long_offsets` = uint64_t[n+1]
// (key i = data[off[i], off[i+1]), length 1..255), `lengths` unused.
int build_host_layout(uint32_t kind, const void* data, const uint8_t* lengths, const uint64_t* values,
                      uint64_t n, uint32_t lut_bytes, HostLayout& out, const uint64_t* long_offsets = nullptr);

// Multi-threaded CPU walk over the flat layout (§4.2, Fig. 7).
void host_layout_lookup(const HostLayout& L, uint32_t kind, const void* queries, const uint8_t* lengths,
                        uint64_t n, uint64_t* out, int threads);

// Per-query count of the 32-byte sectors the GPU lookup reads (algorithmic bytes).
void host_layout_sectors(const HostLayout& L, uint32_t kind, const void* queries, const uint8_t* lengths,
                         uint64_t n, uint32_t* sectors, int threads, bool wide = false, uint32_t skip_d = 0);

}  // namespace cuart
