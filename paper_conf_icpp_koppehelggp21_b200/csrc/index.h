// index.h — internal: the device index handle shared by the C ABI translation
// units (capi.cu: single-GPU hot path; dist.cu: the multi-GPU layer).  Not part of
// the public ABI (include/cuart.h).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <mutex>
#include <utility>
#include <vector>

#include "../../include/cuart.h"
#include "builder.h"
#include "kernels.cuh"

using cuart::DevIndex;
using cuart::HostLayout;

struct cuart_layout {
    HostLayout L;
};

// host-buffer pipelines (cuart_lookup_host / cuart_update_host)
static constexpr size_t kStageChunk = size_t(1) << 23;   // ops per pipeline chunk (env CUART_STAGE_CHUNK overrides)
static constexpr int kStages = 4;                          // chunks in flight (streams / staging sets)

struct DistState;   // dist.cu

struct cuart_index {
    int device = 0;
    int num_sms = 148;
    uint32_t key_kind = 0;
    uint32_t lut_bytes = 0;
    uint64_t root = 0;
    uint64_t count[8] = {0};
    uint64_t n_keys = 0;
    uint32_t max_depth = 0;
    uint8_t* arena = nullptr;          // all record buffers + winner words + LUT + error flag
    size_t arena_bytes = 0;
    uint64_t off[8] = {0};
    uint64_t lut_off = 0, winner_off = 0, err_off = 0;
    uint64_t total_leaves = 0;
    DevIndex dix{};
    DevIndex dix_links{};              // dix reading the 8-B LINKS root table (bucketed walks; §5)
    uint32_t epoch = 0;                // update batch epoch (high half of winner words)
    // stream-ordered scratch of every call (bucketing, update stage 1 -> 2 leaf links)
    // comes from this per-index pool: no cudaMalloc / implicit device synchronisation
    // on the hot path, released in cuart_destroy
    cudaMemPool_t pool = nullptr;
    bool hold_epoch = false;           // dist updates: every chunk of a batch shares one epoch
    // l2_persist (§3.2.2): persisting access-policy window over the root tables
    void* l2_base = nullptr;
    size_t l2_bytes = 0;
    float l2_hit = 0.f;
    DistState* dist = nullptr;         // multi-GPU state (cuart_dist_build), else nullptr
    uint64_t free_off = 0;             // free-leaf list (u32 ids) + its counter
    uint64_t llen_off = 0;             // BYTES: key length of every leaf (global leaf id order)
    // host-pipeline staging
    void* stage[4] = {nullptr, nullptr, nullptr, nullptr};
    uint64_t* stage_out[4] = {nullptr, nullptr, nullptr, nullptr};
    uint8_t* stage_len[4] = {nullptr, nullptr, nullptr, nullptr};
    uint64_t* stage_val[4] = {nullptr, nullptr, nullptr, nullptr};
    size_t stage_cap = 0;
    cudaStream_t streams[4] = {nullptr, nullptr, nullptr, nullptr};   // host-pipeline streams
    cudaStream_t ustream = nullptr;                                   // update pipeline: the kernels, in op order
    cudaEvent_t ev_join = nullptr;                                    // host pipelines start after the legacy stream
    cudaEvent_t ev_copied[4] = {nullptr, nullptr, nullptr, nullptr};  // staging set s filled
    cudaEvent_t ev_free[4] = {nullptr, nullptr, nullptr, nullptr};    // staging set s consumed
    int policy = 5;                    // cache-policy variant of the kernels (kernels.cuh Loader)
    uint32_t lut_format = CUART_LUT_LINKS;
    uint64_t lutc_off = 0;             // compact / rank LUT region
    uint64_t lutw_off = 0;             // wide LUT region (32 B/entry), 0 bytes if absent
    uint64_t skip_off = 0;             // skip table region (byte strings), 0 bytes if absent
    uint32_t skip_d = 0;               // its prefix length (0: no table)
    uint64_t skip_entries = 0;         // its slots
    bool wide = false;
    uint64_t lut_exceptions = 0;       // RANK: entries served by the 64-bit table
    int grid_ctas_per_sm = 0;          // 0 = default grid (one op per thread); else persistent grid
    bool ktimer = false;               // record CUDA events around every k_lookup launch
    int ilp = 2;                       // queries per thread of the pre-bucketed wide walk (k_lookup_wq)
    unsigned wq_tpb = 64;              // k_lookup_wq threads per CTA (CUART_WQ_TPB: 32 / 64 / 128 / 256)
    unsigned lk_tpb = 256;             // k_lookup threads per CTA (CUART_LOOKUP_TPB: 64 / 128 / 256)
    unsigned upd2_tpb = 256;           // k_upd2 threads per CTA (CUART_UPD2_TPB: 64 / 256)
    int wq_lp = 3;                     // k_lookup_wq leaf-load cache policy (CUART_WQ_LEAFPOL, kernels.cuh leafv4_b)
    // K-BUCKET on the root byte >> shift: 256 >> shift buckets (CUART_BUCKET_SHIFT).  Set
    // at upload: 64 buckets when a bucket's slice of the walked records stays within
    // 64 MB (c2, c3: runs of ~64 keys per tile cut the run-scattered traffic of scatter
    // and gather while the slice stays L2-resident), else 256 (c5 at N = 1: 60 GB).
    uint32_t bucket_shift = 0;
    std::mutex kmu;
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> kev;
    uint64_t klookups = 0;
    uint64_t kslice = 0;               // timed launches that were k_lookup_slice
    // f4 (CUART_KEY_LONG): host-resident leaves of the keys longer than 32 bytes
    std::vector<uint8_t> long_bytes;
    std::vector<uint64_t> long_off, long_vals;
    uint32_t prebucket = CUART_PREBUCKET_AUTO;   // a5: reorder large lookup batches by bucket (bucket.cuh)
    uint32_t bucket_form = CUART_BUCKET_TILE;    // a5 batch layout: tile-sorted (k_tsort) or global (k_bscatter)
    uint32_t tile_group = 0;                     // tiles per tile-form walk CTA (0 = from the bucket count)
    uint32_t wt_tpb = 0;                         // k_lookup_wt CTA size (0: 64 integer, 256 byte strings; knob CUART_WT_TPB)
    uint32_t tsort_vec = 1;                      // k_tsort with 16-B key loads when the batch is 16-B aligned (knob CUART_TSORT_VEC)
    uint32_t tsort_b1k = 0;                      // byte-string tile sort: 1024 threads, keys in registers (knob CUART_TSORT_B1K)
    uint32_t wt_minb = 20;                       // k_lookup_wt min CTAs/SM (register cap; A/B knob CUART_WT_MINB: 1, 20, 24)
    uint32_t slice_lut = CUART_SLICE_AUTO;       // bucketed walk with the bucket's LUT slice in smem
    bool slice_ok = false;                       // RANK table, integer keys, root branch depth + 2 <= k
    uint64_t slice_e0 = 0;                       // common prefix C << 8(k - d): first entry of bucket 0's slice
    uint32_t slice_shift = 0;                    // log2(entries per slice) = 8(k - 1 - d)
    int slice_grid = 0;                          // persistent grid (CTAs) of k_lookup_slice

};


extern std::atomic<uint64_t> g_cuart_launches;

// internal launchers (capi.cu), all asynchronous on stream s
cuart_status launch_lookup(const cuart_index* h, uint32_t kind, const void* q, const uint8_t* lens, uint64_t n,
                           uint64_t* out, cudaStream_t s, const cuart::SegOut* so = nullptr);
cuart_status launch_lookup_direct(const cuart_index* h, uint32_t kind, const void* q, const uint8_t* lens,
                                  uint64_t n, uint64_t* out, cudaStream_t s, const cuart::SegOut* so = nullptr,
                                  bool bucketed = false);
// mode: 0 = updates only, 1 = mixed (is_delete[i]), 2 = all deletes; opidx = priority of
// every op (nullptr = position); with h->hold_epoch the call joins the current epoch;
// keep_leafref (device u64[n], optional) receives the stage-1 leaf links.
cuart_status launch_update(cuart_index* h, uint32_t kind, const void* k, const uint8_t* lens,
                           const uint64_t* vals, const uint8_t* is_delete, int mode, uint64_t n,
                           cudaStream_t s, const uint32_t* opidx = nullptr, bool bucketed = false,
                           uint64_t* keep_leafref = nullptr);
cuart_status dispatch_update(cuart_index* h, const void* k, const uint8_t* lens, const uint64_t* vals, uint64_t n,
                             cudaStream_t s);
// stream-ordered scratch from the index's own memory pool (never synchronises)
cuart_status scratch_alloc(const cuart_index* h, void** p, size_t bytes, cudaStream_t s);
void scratch_free(const cuart_index* h, void* p, cudaStream_t s);
// begin a new update epoch (conflict words of earlier batches become stale, a9)
cuart_status next_epoch(cuart_index* h, cudaStream_t s);
void dist_teardown(cuart_index* h);   // dist.cu: collective teardown of a multi-GPU index
