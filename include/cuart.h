/*
 * cuart.h — C ABI of the B200-native CuART hot path.
 *
 * CuART (Koppehel, Pionteck, Groth, Groppe; ICPP'21).  Citations "P:<n>" are
 * line numbers of the paper text with the section they fall in.
 *
 *  - cuart_build   : populate + map a host ART into the per-node-type device
 *                    buffers (§4.1 "Populating the ART index /
 *                    Mapping the CPU ART into the buffer structure"; layout
 *                    P:108-110 §3.2.1; root lookup table P:112/§3.2.2).
 *  - cuart_lookup  : batched exact-match lookups on the GPU (Fig. 3, P:98;
 *                    P:108 §3.2.1).
 *  - cuart_update  : batched in-place value replacement, two stages with
 *                    highest-op-index-wins conflict resolution (P:141-143
 *                    §3.4, Fig. 6).
 *  - cuart_destroy : free everything the library owns.
 *
 * Conventions (all calls):
 *  - Every call returns cuart_status; no C++ exception crosses the ABI.
 *  - Keys: CUART_KEY_U64 = uint64_t[n] and CUART_KEY_U32 = uint32_t[n] in the
 *    machine's native byte order; the library orders them numerically (they
 *    are indexed as big-endian byte strings, the binary-comparable form of
 *    ART [17]).  CUART_KEY_BYTES = n slots of CUART_MAX_KEY (32) bytes plus
 *    lengths[n] in [1, 32]; bytes past the length are ignored.  The maximum key
 *    length is the paper's compile-time constant (§3.2.1).  A byte-string
 *    key set must be prefix-free (no stored key is a proper prefix of another).
 *  - Values are uint64_t.  CUART_MISS (UINT64_MAX) is the lookup result for
 *    an absent key and is therefore reserved: it may not be stored.
 *  - Ownership: the caller owns every input/output buffer; the library owns
 *    the index arena and its scratch and frees them in cuart_destroy.
 *  - Pointers: cuart_build takes HOST pointers and is synchronous.
 *    cuart_lookup / cuart_update take DEVICE pointers (on the index's device),
 *    only enqueue work on `stream` (a cudaStream_t passed as void*, NULL =
 *    legacy default stream) and never synchronise the host.
 *    cuart_lookup_host / cuart_update_host take HOST pointers (pinned for full
 *    speed) and run a chunked H2D -> kernel -> D2H pipeline on the index's own
 *    streams; they start after every operation already queued on the legacy
 *    default stream (and so on every blocking stream) -- work on other
 *    non-blocking streams must be synchronised by the caller -- and return when
 *    the results are in host memory.
 *  - Ordering: lookups may run concurrently on several streams; updates on
 *    one index must not overlap each other (the conflict scratch is per index).
 *    A lookup concurrent with an update sees the old or the new 8-byte value
 *    ("atomically replace values", §1.1) — outside parity guarantees.
 *  - n == 0 is a no-op returning CUART_OK.
 */
#ifndef CUART_H
#define CUART_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define CUART_MAX_KEY 32
#define CUART_MISS UINT64_MAX

typedef enum {
    CUART_OK = 0,
    CUART_ERR_INVALID_ARGUMENT = 1, /* NULL with n > 0, bad kind, bad option    */
    CUART_ERR_KEY_LENGTH = 2,       /* key length 0 or > 32                      */
    CUART_ERR_NOT_PREFIX_FREE = 3,  /* build: a key is a proper prefix of another */
    CUART_ERR_RESERVED_VALUE = 4,   /* build: value == CUART_MISS; update: sticky */
    CUART_ERR_OOM = 5,              /* host or device allocation failed          */
    CUART_ERR_CUDA = 6,             /* a CUDA runtime call / launch failed        */
    CUART_ERR_NCCL = 7,             /* reserved for the multi-GPU layer          */
    CUART_ERR_NO_DEVICE = 8,        /* no CUDA device / wrong device             */
    CUART_ERR_TOO_LARGE = 9,        /* a node buffer exceeds the 52-bit link index */
    CUART_ERR_INTERNAL = 10
} cuart_status;

typedef enum { CUART_KEY_U32 = 1, CUART_KEY_U64 = 2, CUART_KEY_BYTES = 3,
               CUART_KEY_LONG = 4 /* f4: 1..255-byte keys, only through the *_long calls */ } cuart_key_kind;

typedef struct {
    cuart_key_kind kind;
    const void* data;        /* U32: uint32_t[n]; U64: uint64_t[n]; BYTES: uint8_t[n][32] */
    const uint8_t* lengths;  /* BYTES only: lengths[n] in [1,32]; NULL otherwise          */
} cuart_keys;

/* Build options.  Zero-initialised = defaults.  All of them change performance
 * only, never results. */
typedef struct {
    uint32_t lut_bytes;          /* 0..3: dense root lookup table over the first k key bytes
                                    (§3.2.2, 2^(8k) links; k=3 -> 128 MiB).
                                    CUART_LUT_AUTO (0xFFFFFFFF) = library choice.          */
    uint32_t l2_persist;         /* 1: a persisting L2 access-policy window (cudaAccessPolicyWindow,
                                    hitRatio 1) over the root lookup table the walks start from
                                    (§3.2.2: the merged upper layers are what the cache
                                    should keep), set on the caller's stream of every call.  It
                                    changes performance only.                                 */
    int32_t device;              /* CUDA device ordinal; -1 = current device                */
    uint32_t lut_format;         /* device form of the root table ("compacted pointers"):
                                    CUART_LUT_FORMAT_AUTO, CUART_LUT_LINKS (8-B links),
                                    CUART_LUT_COMPACT32 (4-B entries), CUART_LUT_RANK (32-B
                                    blocks per 32 entries: type bit-planes + per-type base
                                    index + rank; 1 B/entry, sized for L2 residency).
                                    COMPACT32 / RANK need integer keys (else LINKS).        */
    uint32_t prebucket;          /* query pre-bucketing of large lookup batches (§8(a) a5):
                                    CUART_PREBUCKET_AUTO (on for integer-key batches of
                                    >= 2^22 ops, lookups and plain updates),
                                    CUART_PREBUCKET_OFF, CUART_PREBUCKET_ON.  Results are
                                    identical; it reorders the batch so concurrent warps
                                    share subtrees (stream-ordered scratch from the index's pool: ~19 B per u64
                                    query in the tile form, ~18 B in the global form). */
    uint32_t slice_lut;          /* pre-bucketed lookups with a RANK root table: every
                                    CTA walks its share of each bucket with the bucket's slice
                                    of the table staged in shared memory (64 KiB at k=3),
                                    so the first access of a walk is not an L2 request.
                                    CUART_SLICE_AUTO (= off: measured slower on B200, the
                                    slices take L1 capacity), CUART_SLICE_OFF,
                                    CUART_SLICE_ON.  Results are identical.                */
    uint32_t wide_lut;           /* pre-bucketed walks start from a wide root table: 32 B per
                                    entry = the link + the sorted keys of the N4 / N16 it
                                    points to ("merged top layers"), so the first
                                    node's key read is skipped, + the node's leaf run (when
                                    all its children are leaves they are consecutive in the
                                    ordered leaf buffer, so child i = run + i and the
                                    child-link read is skipped too; for a full N256 of
                                    leaves child b = run + b).  CUART_WIDE_AUTO (on when
                                    most entries lead to an N4/N16 or a full N256 of
                                    leaves), CUART_WIDE_OFF, CUART_WIDE_ON.  Results are
                                    identical.                                             */
    uint32_t bucket_form;        /* layout of a pre-bucketed integer-key lookup batch (a5):
                                    CUART_BUCKET_TILE sorts every 4096-query tile by bucket in
                                    place and walks bucket b's runs of all tiles together
                                    (no histogram pass, no global scatter: 52 streaming B per
                                    u64 query); CUART_BUCKET_GLOBAL scatters the batch into
                                    one contiguous run per bucket (60 B per query).
                                    CUART_BUCKET_FORM_AUTO = tile.  Byte-string batches
                                    (bucketed only with CUART_PREBUCKET_ON) take the tile
                                    form too; multi-GPU owner walks (fused return) and
                                    update batches use the global form.  Results are
                                    identical.                                             */
    uint32_t skip_log2;          /* byte-string indexes: skip table over the first D key bytes
                                    ("merged upper layers", where the first bytes do not
                                    discriminate): D = the longest prefix (<= 16 B) with at most
                                    2^skip_log2 distinct values among the keys; a lookup starts at
                                    the node covering its D-byte prefix.  0 = library choice
                                    (2^20: table <= 64 MB, L2-resident); 1..26 explicit; the
                                    env CUART_SKIP=0 disables it.  Results are identical.     */
} cuart_build_opts;
#define CUART_BUCKET_FORM_AUTO 0u
#define CUART_BUCKET_GLOBAL 1u
#define CUART_BUCKET_TILE 2u
#define CUART_WIDE_AUTO 0u
#define CUART_WIDE_OFF 1u
#define CUART_WIDE_ON 2u
#define CUART_SLICE_AUTO 0u
#define CUART_SLICE_OFF 1u
#define CUART_SLICE_ON 2u
#define CUART_PREBUCKET_AUTO 0u
#define CUART_PREBUCKET_OFF 1u
#define CUART_PREBUCKET_ON 2u
#define CUART_LUT_FORMAT_AUTO 0u
#define CUART_LUT_LINKS 1u
#define CUART_LUT_COMPACT32 2u
#define CUART_LUT_RANK 3u
#define CUART_LUT_AUTO 0xFFFFFFFFu

/* Per-node-type counts and bytes of an index (type codes P:108). */
typedef struct {
    uint64_t count[8];           /* [1]=N4 [2]=N16 [3]=N48 [4]=N256 [5]=leaf8 [6]=leaf16 [7]=leaf32 */
    uint64_t bytes[8];
    uint64_t n_keys;
    uint64_t lut_entries;        /* 2^(8*lut_bytes) or 0 */
    uint64_t lut_bytes_total;
    uint64_t arena_bytes;        /* device bytes held by the index (arena + LUT + scratch) */
    uint32_t lut_bytes;
    uint32_t key_kind;
    uint64_t root;               /* packed root link */
    uint32_t max_depth;          /* longest root-to-leaf node chain */
    uint32_t lut_format;         /* CUART_LUT_* in use on the device */
    uint64_t lut_exceptions;     /* RANK: entries served by the 64-bit link table */
    uint32_t wide_lut;           /* 1: pre-bucketed walks start from the wide root table */
    uint64_t l2_window_bytes;    /* l2_persist: bytes under the persisting access-policy window */
    uint32_t skip_prefix;        /* byte strings: prefix length D of the skip table (0 = none) */
    uint64_t skip_slots;         /* its slots (32 B each; at most half of them used)          */
} cuart_stats_t;

typedef struct cuart_index cuart_index;    /* device-resident index (opaque) */
typedef struct cuart_layout cuart_layout;  /* host-resident flattened layout (opaque) */

/* Read-only view of a host layout's arrays. */
typedef struct {
    const uint8_t* buf[8];       /* [1..7] raw records of each type, index order     */
    uint64_t count[8];
    uint64_t record_bytes[8];    /* 64, 160, 672, 2080, 16, 32, 48                   */
    const uint64_t* lut;         /* NULL if lut_bytes == 0                            */
    uint64_t lut_entries;
    uint64_t root;
    uint32_t lut_bytes;
    uint32_t key_kind;
    uint64_t n_keys;
} cuart_layout_view;

/* ---- the hot path -------------------------------------------------------- */
cuart_status cuart_build(const cuart_keys* keys, const uint64_t* values, size_t n,
                         const cuart_build_opts* opts, cuart_index** out);
cuart_status cuart_lookup(const cuart_index* h, const cuart_keys* queries, size_t n,
                          uint64_t* out, void* stream);
cuart_status cuart_update(cuart_index* h, const cuart_keys* keys, const uint64_t* new_values,
                          size_t n, void* stream);
cuart_status cuart_destroy(cuart_index* h);   /* NULL ok */

/* Non-structural device-side deletes (§8(f) f1; §3.3, §3.4: "updates
 * and nonstructural modifying deletes ... use the same implementation ...
 * signaling a deletion through a nil pointer").  cuart_update_ex takes a mixed
 * batch (is_delete[i] != 0 marks op i as a delete; device uint8_t[n]);
 * cuart_erase deletes every key of the batch.  Semantics (reading C17): every op
 * locates its key in the state before the batch; per located key the op with the
 * highest index decides — store its value, or delete.  A delete unlinks the leaf
 * from its parent's child slot (nodes are not collapsed), overwrites the leaf's
 * value with the tombstone CUART_MISS (key bytes stay, so the leaf buffer keeps
 * its lexicographic order) and pushes the leaf id (leaf8 ids, then leaf16, then
 * leaf32) onto the free-leaf list.  Ops on absent or deleted keys are no-ops. */
cuart_status cuart_update_ex(cuart_index* h, const cuart_keys* keys, const uint64_t* new_values,
                             const uint8_t* is_delete, size_t n, void* stream);
cuart_status cuart_erase(cuart_index* h, const cuart_keys* keys, size_t n, void* stream);
/* Range queries (§8(f) f2; §3.2.1: leaves are strictly ordered inside each
 * leaf buffer, so a range is handed back as start and end indices into the leaf
 * arrays).  For query i with inclusive bounds [lo[i], hi[i]]:
 *   bounds[6*i + 2*(c-5)]     = number of class-c leaves with key <  lo[i]
 *   bounds[6*i + 2*(c-5) + 1] = number of class-c leaves with key <= hi[i]
 * for c = 5 (leaf8), 6 (leaf16), 7 (leaf32); the matching leaves are the records
 * [start, end) of that buffer (cuart_dump).  Deleted leaves stay in place with
 * the tombstone value CUART_MISS.  Every key kind: integer keys live in the leaf8
 * buffer; byte strings in all three classes, ordered lexicographically (a proper
 * prefix first; bound bytes past their length are ignored).  Device pointers, bounds
 * uint64_t[6n]; async. */
cuart_status cuart_range(const cuart_index* h, const cuart_keys* lo, const cuart_keys* hi, size_t n,
                         uint64_t* bounds, void* stream);
/* Synchronous read of the free-leaf list: *count entries exist; up to cap copied to ids (host). */
cuart_status cuart_free_leaves(const cuart_index* h, uint32_t* ids, size_t cap, size_t* count);

/* Host-buffer variants: chunked, stream-pipelined H2D -> kernel -> D2H (P:151
 * §4.1: batches, several command streams).  Synchronous. */
cuart_status cuart_lookup_host(const cuart_index* h, const cuart_keys* queries, size_t n,
                               uint64_t* out);
cuart_status cuart_update_host(cuart_index* h, const cuart_keys* keys, const uint64_t* new_values,
                               size_t n);

/* ---- introspection ------------------------------------------------------- */
cuart_status cuart_stats(const cuart_index* h, cuart_stats_t* out);
/* Synchronous device->host copy of every array (a snapshot; P:102 the buffers
 * are regenerated from the host ART).  Free with cuart_layout_free. */
cuart_status cuart_dump(const cuart_index* h, cuart_layout** out);
/* Sticky device-side error flag (e.g. an update carried CUART_MISS); reading
 * synchronises the index's device and clears the flag. */
cuart_status cuart_get_error(cuart_index* h);
const char* cuart_status_string(cuart_status s);
/* Measurement hooks: while enabled, CUDA events bracket every k_lookup launch of
 * this index on its stream; cuart_kernel_time sums their elapsed times (and
 * launch / lookup counts) since the timer was (re)enabled, then resets. */
cuart_status cuart_kernel_timer(cuart_index* h, int enable);
cuart_status cuart_kernel_time(cuart_index* h, double* total_ms, uint64_t* launches, uint64_t* lookups);
/* As cuart_kernel_time; slice_launches = how many of the timed launches were the
 * bucketed walk with the shared-memory root-table slice (k_lookup_slice). */
cuart_status cuart_kernel_time_ex(cuart_index* h, double* total_ms, uint64_t* launches, uint64_t* lookups,
                                  uint64_t* slice_launches);
/* Test hook: set the update epoch (the high half of the per-leaf conflict words,
 * §8(a) a9) so that the wrap path -- every 2^32 - 2 update batches the words are
 * cleared and the epoch restarts at 1 -- can be exercised.  Synchronous. */
cuart_status cuart_debug_set_epoch(cuart_index* h, uint32_t epoch);
/* Kernel launches issued by this library since load (for launch accounting). */
uint64_t cuart_launch_count(void);

/* ---- host layout (no GPU needed) ----------------------------------------- */
/* The canonical ART of the key set flattened into the per-type buffers
 * (one buffer per node type, packed 64-bit type+index links; P:110:
 * fixed-size leaves of 8/16/32-byte keys in lexicographic order). */
cuart_status cuart_layout_build(const cuart_keys* keys, const uint64_t* values, size_t n,
                                const cuart_build_opts* opts, cuart_layout** out);
cuart_status cuart_layout_view_get(const cuart_layout* l, cuart_layout_view* out);
/* CPU lookup engine over the flat layout (§4.2, Fig. 7: the CuART
 * layout used by a multi-threaded CPU lookup).  A separate engine, never a
 * fallback of cuart_lookup. */
cuart_status cuart_layout_lookup(const cuart_layout* l, const cuart_keys* queries, size_t n,
                                 uint64_t* out, int threads);
/* Per-query number of distinct 32-byte sectors the GPU lookup kernel reads on the
 * path of each query (the algorithmic traffic behind the roofline numbers;
 * DESIGN.md "Roofline").  sectors: host uint32_t[n]. */
cuart_status cuart_layout_sectors(const cuart_layout* l, const cuart_keys* queries, size_t n,
                                  uint32_t* sectors, int threads);
/* As cuart_layout_sectors for the walk of a given variant: flags CUART_SECTORS_WIDE =
 * the pre-bucketed walk starting from the wide root table (cuart_build_opts.wide_lut);
 * CUART_SECTORS_SKIP(D) = byte-string walks starting from a skip table over D-byte
 * prefixes (one 32-B probe, then the walk below the covering node; cuart_stats
 * skip_prefix gives D). */
#define CUART_SECTORS_WIDE 1u
#define CUART_SECTORS_SKIP(d) ((uint32_t)(d) << 8)
cuart_status cuart_layout_sectors_ex(const cuart_layout* l, const cuart_keys* queries, size_t n,
                                     uint32_t* sectors, int threads, uint32_t flags);
cuart_status cuart_upload(const cuart_layout* l, const cuart_build_opts* opts, cuart_index** out);
cuart_status cuart_layout_free(cuart_layout* l);  /* NULL ok */

/* ---- multi-GPU routing (range-partitioned mode) ------------ */
/* The key space is split by nparts-1 ascending splitters over the first 8 key
 * bytes read big-endian (U64: the key; U32: key << 32; BYTES: the first 8 bytes,
 * zero padded): owner(k) = number of splitters <= prefix8(k).  cuart_route
 * scatters a batch into per-owner contiguous runs, STABLE in op order (so an
 * owner that receives all sources' runs concatenated by source rank sees the ops
 * in global rank-major order, which is what the update rule needs), and
 * writes perm[i] = the slot of op i.  All pointers are DEVICE pointers on one
 * device; async on `stream`.
 *   splitters  : uint64_t[nparts-1] (device), nparts in [1, 64]
 *   values     : uint64_t[n] or NULL (then send_values is not written)
 *   send_keys  : same element layout as keys->data (8 / 4 / 32 B per key), n slots
 *   send_lengths: BYTES only, uint8_t[n]
 *   perm       : uint32_t[n];  counts: uint64_t[nparts] ops per owner
 *   scratch    : cuart_route_scratch_bytes(n, nparts) bytes
 * n must be < 2^32.  cuart_unroute gathers out[i] = in[perm[i]]. */
size_t cuart_route_scratch_bytes(size_t n, uint32_t nparts);
cuart_status cuart_route(const cuart_keys* keys, size_t n, const uint64_t* splitters, uint32_t nparts,
                         const uint64_t* values, void* send_keys, uint8_t* send_lengths, uint64_t* send_values,
                         uint32_t* perm, uint64_t* counts, void* scratch, void* stream);
cuart_status cuart_unroute(const uint64_t* in, const uint32_t* perm, size_t n, uint64_t* out, void* stream);
/* Stable two-way split of a batch by a per-op flag (device uint8_t[n]): ops with
 * flag 0 first, then flag != 0, each in op order; perm/counts/scratch as for
 * cuart_route with nparts = 2.  Used to split a mixed lookup/update round
 * (reading C7) into its lookups and its updates. */
cuart_status cuart_partition_by_flag(const cuart_keys* keys, size_t n, const uint8_t* flags, const uint64_t* values,
                                     void* out_keys, uint8_t* out_lengths, uint64_t* out_values, uint32_t* perm,
                                     uint64_t* counts, void* scratch, void* stream);

/* ---- keys longer than 32 bytes (§8(f) f4; §3.2.3, option 2) ----------
 * An index of kind CUART_KEY_LONG holds prefix-free byte-string keys of 1..255
 * bytes.  Its inner nodes and the leaves of keys of <= 32 bytes live on the
 * device as usual; the leaves of longer keys live in a HOST leaf buffer, and the
 * device node buffers hold links of type 8 (host leaf) to them.  A GPU walk that
 * reaches such a link signals the host "compare the complete key against host
 * leaf #idx" ("it sets a specific signal in the return value indicating
 * that the CPU needs to compare the complete key along with the address of the
 * actual leaf in main memory"); the library finishes those compares on the host.
 * Keys and queries are packed: key i = data[offsets[i], offsets[i+1]) (HOST
 * pointers, offsets uint64_t[n+1]).  All three calls are synchronous.
 *   cuart_build_long  : as cuart_build (duplicates: last wins; not prefix-free ->
 *                       CUART_ERR_NOT_PREFIX_FREE; length 0 or > 255 -> KEY_LENGTH)
 *   cuart_lookup_long : out[i] = value or CUART_MISS (host uint64_t[n])
 *   cuart_update_long : sequential batch semantics as cuart_update: the
 *                       device leaves by the two-stage kernels, the host leaves
 *                       by the host in op order; absent keys are no-ops.
 * The other calls reject a CUART_KEY_LONG index with CUART_ERR_INVALID_ARGUMENT. */
cuart_status cuart_build_long(const uint8_t* data, const uint64_t* offsets, const uint64_t* values, size_t n,
                              const cuart_build_opts* opts, cuart_index** out);
cuart_status cuart_lookup_long(cuart_index* h, const uint8_t* data, const uint64_t* offsets, size_t n,
                               uint64_t* out, void* stream);
cuart_status cuart_update_long(cuart_index* h, const uint8_t* data, const uint64_t* offsets,
                               const uint64_t* values, size_t n, void* stream);

/* out[i] = CUART_MISS for i < n (device pointer; async): the result slots of ops that
 * return no lookup value (the update ops of a mixed round, reading C7). */
cuart_status cuart_fill_miss(uint64_t* out, size_t n, void* stream);

/* ---- multi-GPU index: one process per GPU of one box --------
 * The paper runs one GPU (§4.1 mentions a 2-GPU server only as hardware);
 * the multi-GPU layer is the north star's scaling of its batched lookups and
 * updates (§4.1: batches, several command streams) over NVLink/NVSwitch.
 *
 * Modes:
 *   CUART_DIST_RANGE   : the key space is range-partitioned over the first 8 key
 *                        bytes read big-endian (nranks-1 ascending splitters; owner(k)
 *                        = number of splitters <= prefix8(k)).  Every rank indexes its
 *                        range; a batch is routed to the owners, served there and the
 *                        results routed back (K-ROUTE fused with K-BUCKET: the source's
 *                        pre-bucketing partitions by (owner, owner's bucket), so every
 *                        owner receives runs that are already bucketed for its walk).
 *   CUART_DIST_REPLICA : every rank holds the full index; lookups are served locally
 *                        with no exchange; update batches are exchanged and applied by
 *                        every rank, so the replicas stay bit-identical.
 * Transports:
 *   CUART_TRANSPORT_P2P  : receive windows in device memory exported with CUDA IPC and
 *                        mapped by every peer (NVLink / NVSwitch).  The source's scatter
 *                        kernel stores every op straight into its owner's window, the
 *                        owner's walk stores every result straight into the source's
 *                        result window; cross-rank ordering uses device-side release /
 *                        acquire flags (no host barrier, no stream synchronisation); the
 *                        host only reads the per-chunk count matrix from mapped pinned
 *                        memory to size the owner's launches.  Batches are cut into
 *                        chunks with two window slots in flight, so the routing of chunk
 *                        c+1 overlaps the walk of chunk c.
 *   CUART_TRANSPORT_NCCL : route into a local send buffer, then grouped ncclSend /
 *                        ncclRecv of the runs (and of the results), counts via
 *                        ncclAllGather (the library-collective baseline).
 * Semantics (reading C7): the ops of one cuart_dist_update call are ordered rank-major
 * (all of rank 0's batch, then rank 1's, ...), each rank's batch in its own order; the
 * highest op in that global order wins per key.  Lookups of a call see the
 * state before any later update call.  Results are independent of nranks, mode and
 * transport, and equal a single index updated with the concatenated batches.
 * All dist calls are COLLECTIVE: every rank of the group calls them in the same order
 * (n may differ per rank, including 0).
 */
#define CUART_DIST_REPLICA 1u
#define CUART_DIST_RANGE 2u
#define CUART_TRANSPORT_NCCL 1u
#define CUART_TRANSPORT_P2P 2u
#define CUART_DIST_MAX_RANKS 16
#define CUART_NCCL_ID_BYTES 128
/* Host bootstrap collective: gather `bytes` bytes from every rank into recv
 * (nranks * bytes, rank order).  Returns 0 on success.  Called only inside
 * cuart_dist_build / cuart_destroy / cuart_dist_partition (setup and teardown). */
typedef int (*cuart_allgather_fn)(void* ctx, const void* send, void* recv, size_t bytes);
typedef struct {
    int32_t rank;                 /* this process's rank in [0, nranks)                        */
    int32_t nranks;               /* 1 .. CUART_DIST_MAX_RANKS, one GPU per rank               */
    uint32_t mode;                /* CUART_DIST_RANGE | CUART_DIST_REPLICA                     */
    uint32_t transport;           /* CUART_TRANSPORT_P2P | CUART_TRANSPORT_NCCL                */
    uint8_t nccl_id[CUART_NCCL_ID_BYTES];  /* ncclUniqueId (cuart_dist_unique_id on rank 0, the
                                     same bytes on every rank); unused when transport is P2P and
                                     allgather is set                                          */
    cuart_allgather_fn allgather; /* optional host bootstrap; NULL = ncclAllGather on the comm */
    void* allgather_ctx;
    const uint64_t* splitters;    /* RANGE: nranks-1 ascending host splitters, or NULL = quantiles
                                     of the key set's 8-byte prefixes (identical on every rank)  */
    uint32_t keys_local;          /* RANGE: 1 = keys/values passed to cuart_dist_build are already
                                     this rank's share (splitters required)                    */
    uint32_t reserved0;
    uint64_t chunk;               /* ops per pipeline chunk per rank; 0 = library default       */
    cuart_build_opts opts;        /* the local index (opts.device = this rank's GPU)           */
} cuart_dist_cfg;
/* Writes a fresh ncclUniqueId (CUART_NCCL_ID_BYTES) to id.  Host only. */
cuart_status cuart_dist_unique_id(void* id);
/* Collective build.  keys/values: HOST buffers; RANGE with keys_local = 0 and REPLICA:
 * the global key set, identical on every rank; RANGE with keys_local = 1: this rank's
 * share.  Returns a cuart_index of the local part; cuart_lookup / cuart_update on it act
 * on the local part only; cuart_destroy on it is collective.  Errors as cuart_build,
 * plus CUART_ERR_NCCL (bootstrap / NCCL failure) and CUART_ERR_INVALID_ARGUMENT (bad
 * cfg: rank / nranks / mode / transport, splitters not ascending, ranks disagreeing on
 * the splitters, key kind, window sizes). */
cuart_status cuart_dist_build(const cuart_dist_cfg* cfg, const cuart_keys* keys, const uint64_t* values, size_t n,
                              cuart_index** out);
/* Collective lookup of this rank's batch (DEVICE pointers on this rank's GPU, n may be 0):
 * out[i] = value of queries[i] in the distributed index, else CUART_MISS.  Enqueued on
 * `stream` (internal streams join it); returns after the last chunk's launches are
 * enqueued; n <= 2^32 / nranks. */
cuart_status cuart_dist_lookup(cuart_index* h, const cuart_keys* queries, size_t n, uint64_t* out, void* stream);
/* Collective update: this rank's batch (DEVICE pointers) joins the call's global batch
 * at position rank (reading C7).  Values equal to CUART_MISS are dropped and set the
 * sticky error flag of the owner's index (reading C5).  n <= 2^32 / nranks. */
cuart_status cuart_dist_update(cuart_index* h, const cuart_keys* keys, const uint64_t* new_values, size_t n,
                               void* stream);
/* Collective mixed batch (config 5's rounds, reading C7; RANGE mode): op i is an update
 * iff is_update[i] != 0 (device uint8_t[n]).  Every lookup of the call, on every rank,
 * sees the state before the call; then the call's updates apply in global rank-major
 * order.  out[i] = the lookup result, CUART_MISS for update ops.  One pass per op kind
 * filters the batch itself (no stable partition + inverse permutation).  REPLICA mode
 * returns CUART_ERR_INVALID_ARGUMENT (split the batch with cuart_partition_by_flag). */
cuart_status cuart_dist_mixed(cuart_index* h, const cuart_keys* keys, const uint64_t* values, const uint8_t* is_update,
                              size_t n, uint64_t* out, void* stream);
/* Host-only planning (no GPU): the splitters the build uses (RANGE; nranks-1 entries)
 * and the owner of each key (owner[i], may be NULL).  With a bootstrap in cfg the
 * splitters are all-gathered and compared across ranks (INVALID_ARGUMENT on mismatch). */
cuart_status cuart_dist_partition(const cuart_dist_cfg* cfg, const cuart_keys* keys, size_t n, uint64_t* splitters,
                                  uint8_t* owner);
/* Host-only: the exchange plan of one chunk for rank `me` from the nranks x nranks count
 * matrix M (row-major, M[s*P + o] = ops source s routes to owner o), as the library uses
 * it: seg_start[P+1] (source segments of me's receive window), res_off[P] (first slot of
 * me's results in source s's send order), push_off[P] (first slot of me's run in owner
 * o's window). */
cuart_status cuart_dist_chunk_plan(uint32_t nranks, uint32_t me, const uint64_t* M, uint64_t* seg_start,
                                   uint64_t* res_off, uint64_t* push_off);
/* Statistics of the last dist call on this rank: ops received as owner, chunks. */
cuart_status cuart_dist_last(const cuart_index* h, uint64_t* recv_ops, uint64_t* chunks);

#ifdef __cplusplus
}
#endif
#endif /* CUART_H */
