// dist.cu — the multi-GPU layer behind cuart_dist_* (include/cuart.h; SURVEY §8(b),
// §8(e)).  One process per GPU of one box; every rank holds a local CuART index
// (the global index restricted to its key range, or a full replica).
//
// The paper's path is single-GPU (batched lookups, Fig. 3; two-stage updates
// P:141-143); batching over several command streams is P:151 §4.1.  What this file
// adds is the north star's scaling of that path over NVLink / NVSwitch.
//
// Range mode, transport P2P, one lookup chunk c (slot = c & 1, seq = per-call
// sequence number; S = the source role's stream, O = the owner role's stream):
//   S  K-BUCKET histogram + scan with parts (owner, owner's bucket)     k_bhist, k_bscan_*
//   S  publish this source's per-owner counts into every rank's ctrl    k_publish
//   S  wait for every rank's counts; derive push offsets; copy the
//      count matrix to mapped host memory                               k_wait_counts
//   S  scatter: staged runs stored straight into the owners' windows    k_bscatter<PUSH>
//   S  release "pushed" flags at every owner                            k_signal
//   host  reads the count matrix (mapped memory) to size the owner launches
//   O  acquire every source's "pushed" flag                             k_wait_flags
//   O  wide walk over the received runs (already bucketed by the
//      sources), each result stored into its source's result window    k_lookup_wq<SEG>
//   O  release "results" flags at every source                          k_signal
//   S  acquire every owner's "results" flag, gather into query order    k_wait_flags, k_bgather
// S runs one chunk ahead of the gathers (front(c+1) before back(c)), so the routing
// of chunk c+1 overlaps the walk of chunk c; two window slots are in flight.
// Updates travel with their values and priorities (global rank-major op index,
// reading C7); all chunks of a call share one update epoch at the owner, so the
// highest priority wins per key across chunks.
#include <cuda_runtime.h>
#include <nccl.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <unistd.h>

#include <algorithm>
#include <chrono>
#include <new>
#include <thread>
#include <vector>

#include "bucket.cuh"
#include "index.h"

using namespace cuart;

namespace {

// CUART_DIST_DEBUG=1: trace the host steps of the protocol to stderr
bool dbg_on() {
    static const bool on = getenv("CUART_DIST_DEBUG") != nullptr;
    return on;
}
#define DBG(...)                                  \
    do {                                          \
        if (dbg_on()) {                           \
            fprintf(stderr, "[cuart_dist] " __VA_ARGS__); \
            fputc('\n', stderr);                 \
            fflush(stderr);                       \
        }                                         \
    } while (0)

constexpr uint32_t kMaxRanks = kMaxSeg;            // 16
enum { F_CNT = 0, F_PUSH = 1, F_RES = 2 };
constexpr uint64_t kSpinTimeoutNs = 120ull * 1000000000ull;

// Per-rank control block in device memory, mapped by every peer.
struct Ctrl {
    unsigned long long cnt[3][kMaxRanks][kMaxRanks];   // [slot][source][owner]: rows written by the sources
                                                       // (slots 0/1: chunk parity; 2: the per-call n round)
    unsigned long long flag[3][kMaxRanks];             // [F_*][peer]: sequence numbers (monotonic)
    unsigned int err;                                  // a spin wait timed out
};

struct Peers {
    Ctrl* ctrl[kMaxRanks];
    uint32_t P, me;
};

__device__ __forceinline__ void st_release_sys(unsigned long long* p, unsigned long long v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long ld_relaxed_sys(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint64_t globaltimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// Thread-local spin until *p >= seq (acquire); false on timeout.
__device__ bool spin_ge(const unsigned long long* p, unsigned long long seq) {
    const uint64_t t0 = globaltimer();
    while (ld_acquire_sys(p) < seq) {
        __nanosleep(128);
        if (globaltimer() - t0 > kSpinTimeoutNs) return false;
    }
    return true;
}

// This source's per-owner counts of chunk `seq` into every rank's ctrl (itself
// included), then the CNT flag.  Range: row[o] = ops of o's parts (send-order bases);
// replica: row[o] = m for every o.  One thread per destination rank.
__global__ void k_publish(Peers pe, uint32_t slot, const unsigned int* __restrict__ bases, uint64_t m, uint32_t lbpo,
                          uint32_t replica, unsigned long long seq) {
    const uint32_t o = threadIdx.x;
    if (o >= pe.P) return;
    Ctrl* c = pe.ctrl[o];
    for (uint32_t k = 0; k < pe.P; k++) {
        unsigned long long v = m;
        if (!replica) {                                // bases[kBuckets] = ops staged (a filtered pass stages fewer than m)
            const uint64_t b0 = bases[k << lbpo];
            const uint64_t b1 = k + 1 < pe.P ? uint64_t(bases[(k + 1) << lbpo]) : uint64_t(bases[kBuckets]);
            v = m ? b1 - b0 : 0;
        }
        c->cnt[slot][pe.me][k] = v;
    }
    st_release_sys(&c->flag[F_CNT][pe.me], seq);      // release: the row above is visible first
}

// Wait until every rank published chunk `seq`, then: push adjustment of this source
// per owner (adj[o] = sum over earlier sources of their counts to o, minus o's first
// send-order slot here; replica: the window index w takes the place of o and the send
// order starts at 0), and the count matrix to mapped host memory + its stamp.
__global__ void k_wait_counts(Ctrl* mine, uint32_t P, uint32_t me, uint32_t slot, unsigned long long seq,
                              const unsigned int* __restrict__ bases, uint32_t lbpo, uint32_t replica,
                              long long* __restrict__ adj, unsigned long long* hmat) {
    __shared__ unsigned long long M[kMaxRanks][kMaxRanks];
    __shared__ int ok;
    const uint32_t s = threadIdx.x;
    if (s == 0) ok = 1;
    __syncthreads();
    if (s < P) {
        if (!spin_ge(&mine->flag[F_CNT][s], seq)) ok = 0;
        for (uint32_t o = 0; o < P; o++) M[s][o] = ld_relaxed_sys(&mine->cnt[slot][s][o]);   // after the acquire
    }
    __syncthreads();
    if (!ok) {
        if (s == 0) atomicExch(&mine->err, 1u);
        return;
    }
    if (s < P) {
        unsigned long long off = 0;
        for (uint32_t q = 0; q < me; q++) off += M[q][s];
        const long long first = (replica || P == 1) ? 0ll : (long long)bases[s << lbpo];
        adj[s] = (long long)off - first;
        for (uint32_t o = 0; o < P; o++) hmat[s * P + o] = M[s][o];
    }
    __syncthreads();
    if (s == 0) {
        __threadfence_system();
        *(volatile unsigned long long*)&hmat[P * P] = seq;
    }
}

// Release flag `which` = seq at every rank (this rank's previous kernels in stream
// order wrote the data the flag publishes).
__global__ void k_signal(Peers pe, uint32_t which, unsigned long long seq) {
    const uint32_t o = threadIdx.x;
    if (o >= pe.P) return;
    __threadfence_system();
    st_release_sys(&pe.ctrl[o]->flag[which][pe.me], seq);
}

// Acquire flag `which` >= seq from every rank.
__global__ void k_wait_flags(Ctrl* mine, uint32_t P, uint32_t which, unsigned long long seq) {
    const uint32_t s = threadIdx.x;
    if (s >= P) return;
    if (!spin_ge(&mine->flag[which][s], seq)) atomicExch(&mine->err, 1u);
    __threadfence();
}

// NCCL transport: this source's per-owner counts (row) from the send-order bases.
__global__ void k_row(const unsigned int* __restrict__ bases, uint64_t m, uint32_t P, uint32_t lbpo, uint32_t replica,
                      unsigned long long* __restrict__ row) {
    const uint32_t o = threadIdx.x;
    if (o >= P) return;
    if (replica) {
        row[o] = m;
        return;
    }
    const uint64_t b0 = bases[o << lbpo];
    const uint64_t b1 = o + 1 < P ? uint64_t(bases[(o + 1) << lbpo]) : uint64_t(bases[kBuckets]);
    row[o] = m ? b1 - b0 : 0;
}

struct WinHandle {            // one exported device allocation
    int pid;
    int dev;
    void* ptr;
    unsigned char ipc[sizeof(cudaIpcMemHandle_t)];
};

// Buffers of one rank: the receive window (keys, lengths, values, priorities) and
// the result window (this source's results in send order), two chunk slots each,
// and the control block.  Exported to the peers for transport P2P.
enum { B_KEYS = 0, B_LENS, B_VALS, B_PRIO, B_RES, B_SEND, B_SENDL, B_SENDV, B_SENDP, B_ORES, kNumBuf };

}  // namespace

struct DistState {
    int rank = 0;
    uint32_t P = 1;
    uint32_t mode = CUART_DIST_RANGE, transport = CUART_TRANSPORT_P2P;
    cuart_allgather_fn ag = nullptr;
    void* ag_ctx = nullptr;
    ncclComm_t comm = nullptr;
    OwnerPart part{};
    uint32_t lbpo = 8;
    uint64_t chunk = 0;           // C: ops per chunk per source
    uint64_t wcap = 0;            // receive window capacity per slot: P * C ops
    uint32_t kind = 0;
    size_t ks = 8;
    Ctrl* ctrl = nullptr;
    uint8_t* buf[kNumBuf][2] = {};                 // local allocations
    uint8_t* peer[kNumBuf][2][kMaxRanks] = {};     // peers' windows (P2P), own entry = local
    Ctrl* pctrl[kMaxRanks] = {};
    std::vector<void*> owned;
    std::vector<void*> imported;
    unsigned long long* hmat = nullptr;            // mapped pinned: [3][P*P + 1] (slot as Ctrl::cnt)
    // per-slot source-side bucketing scratch
    unsigned int* hist[2] = {};
    unsigned int* tot[2] = {};
    uint16_t* jpos[2] = {};
    long long* adj[3] = {};
    unsigned long long* row = nullptr;             // NCCL: this source's row
    unsigned long long* mat = nullptr;             // NCCL: all-gathered matrix (device)
    unsigned long long* hrow = nullptr;            // NCCL: pinned host copy of the matrix
    cudaStream_t S = nullptr, O = nullptr;
    cudaEvent_t ev_in = nullptr, ev_o = nullptr, ev_s = nullptr;
    unsigned long long seq = 0;
    uint64_t last_recv = 0, last_chunks = 0;
    bool failed = false;
};

namespace {

size_t key_bytes(uint32_t kind) { return kind == CUART_KEY_U64 ? 8 : kind == CUART_KEY_U32 ? 4 : 32; }

uint64_t prefix8_host(uint32_t kind, const void* data, const uint8_t* lens, size_t i) {
    if (kind == CUART_KEY_U64) return ((const uint64_t*)data)[i];
    if (kind == CUART_KEY_U32) return uint64_t(((const uint32_t*)data)[i]) << 32;
    const uint8_t* s = (const uint8_t*)data + 32 * i;
    uint64_t p = 0;
    for (uint32_t b = 0; b < 8; b++) p = (p << 8) | (b < lens[i] ? s[b] : 0u);
    return p;
}

uint32_t owner_host(const uint64_t* sp, uint32_t nsp, uint64_t p) {
    uint32_t o = 0;
    for (uint32_t j = 0; j < nsp; j++) o += sp[j] <= p ? 1u : 0u;
    return o;
}

uint32_t ceil_log2(uint32_t x) {
    uint32_t l = 0;
    while ((1u << l) < x) l++;
    return l;
}

cuart_status check_cfg(const cuart_dist_cfg* c) {
    if (!c) return CUART_ERR_INVALID_ARGUMENT;
    if (c->nranks < 1 || c->nranks > int32_t(kMaxRanks) || c->rank < 0 || c->rank >= c->nranks)
        return CUART_ERR_INVALID_ARGUMENT;
    if (c->mode != CUART_DIST_RANGE && c->mode != CUART_DIST_REPLICA) return CUART_ERR_INVALID_ARGUMENT;
    if (c->transport != CUART_TRANSPORT_P2P && c->transport != CUART_TRANSPORT_NCCL) return CUART_ERR_INVALID_ARGUMENT;
    if (c->keys_local && (c->mode != CUART_DIST_RANGE || (c->nranks > 1 && !c->splitters)))
        return CUART_ERR_INVALID_ARGUMENT;
    if (c->splitters)
        for (int32_t j = 1; j + 1 < c->nranks; j++)
            if (c->splitters[j] < c->splitters[j - 1]) return CUART_ERR_INVALID_ARGUMENT;
    return CUART_OK;
}

// Quantile splitters of the key set's 8-byte prefixes (deterministic: every rank
// computes the same from the same global key set).
void quantile_splitters(uint32_t kind, const void* data, const uint8_t* lens, size_t n, uint32_t P, uint64_t* sp) {
    if (P <= 1) return;
    if (n == 0) {
        for (uint32_t j = 1; j < P; j++) sp[j - 1] = (~uint64_t(0) / P) * j;
        return;
    }
    std::vector<uint64_t> pre(n);
    for (size_t i = 0; i < n; i++) pre[i] = prefix8_host(kind, data, lens, i);
    std::sort(pre.begin(), pre.end());
    for (uint32_t j = 1; j < P; j++) sp[j - 1] = pre[(uint64_t(j) * n) / P];
}

// Host bootstrap allgather: the caller's callback, else ncclAllGather over the comm.
cuart_status boot_allgather(DistState* d, const void* send, void* recv, size_t bytes) {
    if (d->ag) return d->ag(d->ag_ctx, send, recv, bytes) == 0 ? CUART_OK : CUART_ERR_NCCL;
    if (!d->comm) return d->P == 1 ? (memcpy(recv, send, bytes), CUART_OK) : CUART_ERR_NCCL;
    void* ds = nullptr;
    void* dr = nullptr;
    if (cudaMalloc(&ds, bytes) != cudaSuccess || cudaMalloc(&dr, bytes * d->P) != cudaSuccess) {
        cudaFree(ds);
        return CUART_ERR_OOM;
    }
    cuart_status rc = CUART_OK;
    if (cudaMemcpy(ds, send, bytes, cudaMemcpyHostToDevice) != cudaSuccess) rc = CUART_ERR_CUDA;
    if (rc == CUART_OK && ncclAllGather(ds, dr, bytes, ncclUint8, d->comm, d->S) != ncclSuccess) rc = CUART_ERR_NCCL;
    if (rc == CUART_OK && cudaStreamSynchronize(d->S) != cudaSuccess) rc = CUART_ERR_CUDA;
    if (rc == CUART_OK && cudaMemcpy(recv, dr, bytes * d->P, cudaMemcpyDeviceToHost) != cudaSuccess) rc = CUART_ERR_CUDA;
    cudaFree(ds);
    cudaFree(dr);
    return rc;
}

cuart_status boot_barrier(DistState* d) {
    std::vector<uint8_t> r(d->P);
    uint8_t one = 1;
    return boot_allgather(d, &one, r.data(), 1);
}

cuart_status dalloc(DistState* d, void** p, size_t bytes) {
    *p = nullptr;
    const cudaError_t e = cudaMalloc(p, bytes ? bytes : 256);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return e == cudaErrorMemoryAllocation ? CUART_ERR_OOM : CUART_ERR_CUDA;
    }
    d->owned.push_back(*p);
    return CUART_OK;
}

void free_state(DistState* d) {
    if (!d) return;
    for (void* p : d->imported) cudaIpcCloseMemHandle(p);
    for (void* p : d->owned) cudaFree(p);
    if (d->hmat) cudaFreeHost(d->hmat);
    if (d->hrow) cudaFreeHost(d->hrow);
    if (d->comm) ncclCommDestroy(d->comm);
    if (d->S) cudaStreamDestroy(d->S);
    if (d->O) cudaStreamDestroy(d->O);
    if (d->ev_in) cudaEventDestroy(d->ev_in);
    if (d->ev_o) cudaEventDestroy(d->ev_o);
    if (d->ev_s) cudaEventDestroy(d->ev_s);
    delete d;
}

// Host plan of one chunk (cuart_dist_chunk_plan): M row-major [source][owner].
void chunk_plan(uint32_t P, uint32_t me, const unsigned long long* M, uint64_t* seg_start, uint64_t* res_off,
                uint64_t* push_off) {
    seg_start[0] = 0;
    for (uint32_t s = 0; s < P; s++) seg_start[s + 1] = seg_start[s] + M[s * P + me];
    for (uint32_t s = 0; s < P; s++) {
        uint64_t r = 0;
        for (uint32_t o = 0; o < me; o++) r += M[s * P + o];
        res_off[s] = r;
    }
    for (uint32_t o = 0; o < P; o++) {
        uint64_t p = 0;
        for (uint32_t s = 0; s < me; s++) p += M[s * P + o];
        push_off[o] = p;
    }
}

// Spin (host) until the mapped matrix of `slot` carries stamp `seq`.
cuart_status host_wait_matrix(DistState* d, uint32_t slot, unsigned long long seq) {
    const size_t stride = size_t(d->P) * d->P + 1;
    volatile unsigned long long* stamp = d->hmat + slot * stride + size_t(d->P) * d->P;
    const auto t0 = std::chrono::steady_clock::now();
    uint64_t spins = 0;
    while (*stamp < seq) {
        if (++spins > 1024) std::this_thread::yield();
        if ((spins & 0xFFFF) == 0) {
            if (cudaStreamQuery(d->S) != cudaErrorNotReady && *stamp < seq) {
                // S drained without the stamp: a device wait failed (timeout) or a launch failed
                unsigned int err = 0;
                cudaMemcpy(&err, &d->ctrl->err, 4, cudaMemcpyDeviceToHost);
                if (*stamp < seq) return CUART_ERR_INTERNAL;
            }
            if (std::chrono::steady_clock::now() - t0 > std::chrono::seconds(300)) return CUART_ERR_INTERNAL;
        }
    }
    return CUART_OK;
}

Peers peers_of(const DistState* d) {
    Peers p{};
    for (uint32_t r = 0; r < d->P; r++) p.ctrl[r] = d->pctrl[r];
    p.P = d->P;
    p.me = uint32_t(d->rank);
    return p;
}

#define D_TRY(x)                                                                                   \
    do {                                                                                           \
        cudaError_t e_ = (x);                                                                      \
        if (e_ != cudaSuccess) return e_ == cudaErrorMemoryAllocation ? CUART_ERR_OOM : CUART_ERR_CUDA; \
    } while (0)
#define N_TRY(x)                                  \
    do {                                          \
        if ((x) != ncclSuccess) return CUART_ERR_NCCL; \
    } while (0)

// ---------------------------------------------------------------- source side: K-BUCKET by (owner, bucket)
// Histogram + scans of chunk `slot` of m ops at q (send order = part order).
FilteredOwnerPart filtered(const DistState* d, const uint8_t* flags, uint32_t want) {
    FilteredOwnerPart f;
    static_cast<OwnerPart&>(f) = d->part;
    f.flags = flags;
    f.want = want;
    return f;
}

template <class Key>
cuart_status front_bucket(cuart_index* h, DistState* d, uint32_t slot, const void* q, const uint8_t* lens, uint64_t m,
                          cudaStream_t s, const uint8_t* flags = nullptr, uint32_t want = 0) {
    if (m == 0) return CUART_OK;
    const uint64_t tiles = (m + kBucketTile - 1) / kBucketTile;
    const bool replica = d->mode == CUART_DIST_REPLICA;
    const uint32_t nparts = replica ? uint32_t(kBuckets >> h->bucket_shift) : (d->P << d->lbpo);
    const uint32_t depth = (link_type(h->root) >= T_N4 && link_type(h->root) <= T_N256 ? link_aux(h->root) : 0u) |
                           (h->bucket_shift << 8);
    const bool vec = (uintptr_t(q) & 15) == 0;
    if (replica) {
        if (vec) k_bhist<Key, true><<<unsigned(tiles), kBucketThreads, 0, s>>>(q, lens, m, ByteBucket(depth), d->hist[slot]);
        else k_bhist<Key, false><<<unsigned(tiles), kBucketThreads, 0, s>>>(q, lens, m, ByteBucket(depth), d->hist[slot]);
    } else if (flags) {
        const FilteredOwnerPart fp = filtered(d, flags, want);
        if (vec) k_bhist<Key, true, FilteredOwnerPart><<<unsigned(tiles), kBucketThreads, 0, s>>>(q, lens, m, fp, d->hist[slot]);
        else k_bhist<Key, false, FilteredOwnerPart><<<unsigned(tiles), kBucketThreads, 0, s>>>(q, lens, m, fp, d->hist[slot]);
    } else {
        if (vec) k_bhist<Key, true, OwnerPart><<<unsigned(tiles), kBucketThreads, 0, s>>>(q, lens, m, d->part, d->hist[slot]);
        else k_bhist<Key, false, OwnerPart><<<unsigned(tiles), kBucketThreads, 0, s>>>(q, lens, m, d->part, d->hist[slot]);
    }
    k_bscan_rows<<<nparts, kBucketThreads, 0, s>>>(d->hist[slot], tiles, d->tot[slot]);
    k_bscan<<<1, kBuckets, 0, s>>>(d->tot[slot], nparts);
    g_cuart_launches += 3;
    D_TRY(cudaGetLastError());
    return CUART_OK;
}

// The scatter of chunk `slot`: PUSH into the peers' windows (P2P) or into the local
// send buffer (NCCL).  OPS: values and priorities travel with the keys.
template <class Key, bool OPS>
cuart_status front_scatter(cuart_index* h, DistState* d, uint32_t slot, const void* q, const uint8_t* lens,
                           const uint64_t* vals, uint64_t m, uint32_t prio_base, cudaStream_t s,
                           const uint8_t* flags = nullptr, uint32_t want = 0) {
    if (m == 0) return CUART_OK;
    const uint64_t tiles = (m + kBucketTile - 1) / kBucketTile;
    const bool replica = d->mode == CUART_DIST_REPLICA;
    const uint32_t depth = (link_type(h->root) >= T_N4 && link_type(h->root) <= T_N256 ? link_aux(h->root) : 0u) |
                           (h->bucket_shift << 8);
    const size_t smem = bscatter_smem<Key, OPS>();
    const unsigned T = unsigned(tiles);
    if (d->transport == CUART_TRANSPORT_P2P) {
        PushDst pd{};
        for (uint32_t o = 0; o < d->P; o++) {
            pd.keys[o] = d->peer[B_KEYS][slot][o];
            pd.lens[o] = d->peer[B_LENS][slot][o];
            pd.vals[o] = (uint64_t*)d->peer[B_VALS][slot][o];
            pd.prio[o] = (uint32_t*)d->peer[B_PRIO][slot][o];
        }
        pd.adj = d->adj[slot];
        pd.lbpo = d->lbpo;
        pd.nrep = replica ? d->P : 0;
        if (replica)
            k_bscatter<Key, OPS, ByteBucket, true><<<T, kBucketThreads, smem, s>>>(
                q, lens, m, ByteBucket(depth), d->hist[slot], d->tot[slot], nullptr, nullptr, d->jpos[slot], vals, nullptr,
                nullptr, prio_base, pd);
        else if (flags)
            k_bscatter<Key, OPS, FilteredOwnerPart, true><<<T, kBucketThreads, smem, s>>>(
                q, lens, m, filtered(d, flags, want), d->hist[slot], d->tot[slot], nullptr, nullptr, d->jpos[slot], vals,
                nullptr, nullptr, prio_base, pd);
        else
            k_bscatter<Key, OPS, OwnerPart, true><<<T, kBucketThreads, smem, s>>>(
                q, lens, m, d->part, d->hist[slot], d->tot[slot], nullptr, nullptr, d->jpos[slot], vals, nullptr, nullptr,
                prio_base, pd);
    } else {
        if (replica)
            k_bscatter<Key, OPS, ByteBucket, false><<<T, kBucketThreads, smem, s>>>(
                q, lens, m, ByteBucket(depth), d->hist[slot], d->tot[slot], d->buf[B_SEND][slot], d->buf[B_SENDL][slot],
                d->jpos[slot], vals, (uint64_t*)d->buf[B_SENDV][slot], (uint32_t*)d->buf[B_SENDP][slot], prio_base);
        else if (flags)
            k_bscatter<Key, OPS, FilteredOwnerPart, false><<<T, kBucketThreads, smem, s>>>(
                q, lens, m, filtered(d, flags, want), d->hist[slot], d->tot[slot], d->buf[B_SEND][slot],
                d->buf[B_SENDL][slot], d->jpos[slot], vals, (uint64_t*)d->buf[B_SENDV][slot],
                (uint32_t*)d->buf[B_SENDP][slot], prio_base);
        else
            k_bscatter<Key, OPS, OwnerPart, false><<<T, kBucketThreads, smem, s>>>(
                q, lens, m, d->part, d->hist[slot], d->tot[slot], d->buf[B_SEND][slot], d->buf[B_SENDL][slot],
                d->jpos[slot], vals, (uint64_t*)d->buf[B_SENDV][slot], (uint32_t*)d->buf[B_SENDP][slot], prio_base);
    }
    g_cuart_launches++;
    D_TRY(cudaGetLastError());
    return CUART_OK;
}

template <class Key, bool OPS>
void set_scatter_smem() {
    cudaFuncSetAttribute(k_bscatter<Key, OPS, FilteredOwnerPart, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         int(bscatter_smem<Key, OPS>()));
    cudaFuncSetAttribute(k_bscatter<Key, OPS, FilteredOwnerPart, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         int(bscatter_smem<Key, OPS>()));
    cudaFuncSetAttribute(k_bscatter<Key, OPS, ByteBucket, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         int(bscatter_smem<Key, OPS>()));
    cudaFuncSetAttribute(k_bscatter<Key, OPS, OwnerPart, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         int(bscatter_smem<Key, OPS>()));
    cudaFuncSetAttribute(k_bscatter<Key, OPS, ByteBucket, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         int(bscatter_smem<Key, OPS>()));
    cudaFuncSetAttribute(k_bscatter<Key, OPS, OwnerPart, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         int(bscatter_smem<Key, OPS>()));
}

// ---------------------------------------------------------------- the chunked protocol
struct Call {
    const void* q;
    const uint8_t* lens;
    const uint64_t* vals;     // updates
    uint64_t* out;            // lookups
    uint64_t n;
    bool update;
    const uint8_t* flags = nullptr;   // mixed batch: op i is an update iff flags[i] != 0; this pass
                                      // serves the updates (update) or the lookups (!update) only
};

template <class Key>
cuart_status front(cuart_index* h, DistState* d, const Call& c, uint64_t ci, unsigned long long seq) {
    const uint32_t slot = uint32_t(ci & 1);
    const uint64_t b0 = ci * d->chunk;
    const uint64_t m = b0 < c.n ? std::min<uint64_t>(d->chunk, c.n - b0) : 0;
    const void* q = (const uint8_t*)c.q + b0 * d->ks;
    const uint8_t* l = c.lens ? c.lens + b0 : nullptr;
    const uint8_t* fl = c.flags ? c.flags + b0 : nullptr;
    const uint32_t want = c.update ? 1u : 0u;
    const bool replica = d->mode == CUART_DIST_REPLICA;
    cudaStream_t s = d->S;
    cuart_status rc = front_bucket<Key>(h, d, slot, q, l, m, s, fl, want);
    if (rc != CUART_OK) return rc;
    // tot[slot] holds the send-order bases (k_bscan); an empty chunk has none
    if (m == 0) D_TRY(cudaMemsetAsync(d->tot[slot], 0, (kBuckets + 1) * 4, s));
    const uint32_t prio_base = uint32_t(uint64_t(d->rank) * ((uint64_t(1) << 32) / d->P) + b0);
    if (d->transport == CUART_TRANSPORT_P2P) {
        const Peers pe = peers_of(d);
        k_publish<<<1, 32, 0, s>>>(pe, slot, d->tot[slot], m, d->lbpo, replica ? 1u : 0u, seq);
        k_wait_counts<<<1, 32, 0, s>>>(d->ctrl, d->P, uint32_t(d->rank), slot, seq, d->tot[slot], d->lbpo,
                                       replica ? 1u : 0u, d->adj[slot], d->hmat + slot * (size_t(d->P) * d->P + 1));
        g_cuart_launches += 2;
        D_TRY(cudaGetLastError());
        if (c.update) rc = front_scatter<Key, true>(h, d, slot, q, l, c.vals + b0, m, prio_base, s, fl, want);
        else rc = front_scatter<Key, false>(h, d, slot, q, l, nullptr, m, 0, s, fl, want);
        if (rc != CUART_OK) return rc;
        k_signal<<<1, 32, 0, s>>>(pe, F_PUSH, seq);
        g_cuart_launches++;
        D_TRY(cudaGetLastError());
        return CUART_OK;
    }
    // NCCL: scatter into the local send buffer, then the counts
    if (c.update) rc = front_scatter<Key, true>(h, d, slot, q, l, c.vals + b0, m, prio_base, s, fl, want);
    else rc = front_scatter<Key, false>(h, d, slot, q, l, nullptr, m, 0, s, fl, want);
    if (rc != CUART_OK) return rc;
    k_row<<<1, 32, 0, s>>>(d->tot[slot], m, d->P, d->lbpo, replica ? 1u : 0u, d->row);
    g_cuart_launches++;
    D_TRY(cudaGetLastError());
    N_TRY(ncclAllGather(d->row, d->mat, d->P, ncclUint64, d->comm, s));
    D_TRY(cudaMemcpyAsync(d->hrow, d->mat, size_t(d->P) * d->P * 8, cudaMemcpyDeviceToHost, s));
    D_TRY(cudaStreamSynchronize(s));      // the library-collective baseline: host-visible counts
    return CUART_OK;
}

// Owner role of chunk ci: serve the received runs.  M = the chunk's count matrix.
cuart_status owner(cuart_index* h, DistState* d, const Call& c, uint64_t ci, unsigned long long seq,
                   const unsigned long long* M) {
    const uint32_t slot = uint32_t(ci & 1), P = d->P, me = uint32_t(d->rank);
    uint64_t seg[kMaxRanks + 1], res_off[kMaxRanks], push_off[kMaxRanks];
    chunk_plan(P, me, M, seg, res_off, push_off);
    const uint64_t nr = seg[P];
    d->last_recv += nr;
    const bool p2p = d->transport == CUART_TRANSPORT_P2P;
    cudaStream_t o = p2p ? d->O : d->S;
    const Peers pe = peers_of(d);
    if (p2p) {
        k_wait_flags<<<1, 32, 0, o>>>(d->ctrl, P, F_PUSH, seq);
        g_cuart_launches++;
    } else {
        // grouped send / recv of the runs: source order in the receive window
        const size_t ks = d->ks;
        N_TRY(ncclGroupStart());
        uint64_t sbase = 0;
        for (uint32_t r = 0; r < P; r++) {
            // range: my run for r starts at r's first send-order slot; replica: every
            // rank gets my whole chunk (M[me][r] = m for every r)
            const uint64_t cnt_out = M[me * P + r];
            const uint64_t soff = d->mode == CUART_DIST_REPLICA ? 0 : sbase;
            if (d->mode != CUART_DIST_REPLICA) sbase += cnt_out;
            const uint64_t cnt_in = M[r * P + me];
            if (cnt_out) {
                N_TRY(ncclSend(d->buf[B_SEND][slot] + soff * ks, cnt_out * ks, ncclUint8, int(r), d->comm, o));
                if (d->kind == CUART_KEY_BYTES)
                    N_TRY(ncclSend(d->buf[B_SENDL][slot] + soff, cnt_out, ncclUint8, int(r), d->comm, o));
                if (c.update) {
                    N_TRY(ncclSend(d->buf[B_SENDV][slot] + soff * 8, cnt_out, ncclUint64, int(r), d->comm, o));
                    N_TRY(ncclSend(d->buf[B_SENDP][slot] + soff * 4, cnt_out, ncclUint32, int(r), d->comm, o));
                }
            }
            if (cnt_in) {
                N_TRY(ncclRecv(d->buf[B_KEYS][slot] + seg[r] * ks, cnt_in * ks, ncclUint8, int(r), d->comm, o));
                if (d->kind == CUART_KEY_BYTES)
                    N_TRY(ncclRecv(d->buf[B_LENS][slot] + seg[r], cnt_in, ncclUint8, int(r), d->comm, o));
                if (c.update) {
                    N_TRY(ncclRecv(d->buf[B_VALS][slot] + seg[r] * 8, cnt_in, ncclUint64, int(r), d->comm, o));
                    N_TRY(ncclRecv(d->buf[B_PRIO][slot] + seg[r] * 4, cnt_in, ncclUint32, int(r), d->comm, o));
                }
            }
        }
        N_TRY(ncclGroupEnd());
    }
    const void* wk = d->buf[B_KEYS][slot];
    const uint8_t* wl = d->kind == CUART_KEY_BYTES ? d->buf[B_LENS][slot] : nullptr;
    cuart_status rc = CUART_OK;
    if (c.update) {
        if (nr)
            rc = launch_update(h, d->kind, wk, wl, (const uint64_t*)d->buf[B_VALS][slot], nullptr, 0, nr, o,
                               (const uint32_t*)d->buf[B_PRIO][slot], true);
    } else if (nr) {
        SegOut so{};
        so.nseg = P;
        for (uint32_t s = 0; s <= P; s++) so.start[s] = seg[s];
        for (uint32_t s = 0; s < P; s++)
            so.dst[s] = p2p ? (uint64_t*)d->peer[B_RES][slot][s] + res_off[s] : (uint64_t*)d->buf[B_ORES][slot] + seg[s];
        rc = launch_lookup_direct(h, d->kind, wk, wl, nr, nullptr, o, &so, true);
    }
    if (rc != CUART_OK) return rc;
    if (p2p) {
        k_signal<<<1, 32, 0, o>>>(pe, F_RES, seq);       // results stored / window consumed
        g_cuart_launches++;
        D_TRY(cudaGetLastError());
    } else if (!c.update && d->mode == CUART_DIST_RANGE) {
        // results back: owner sends segment s to source s; source receives owner r's
        // results at r's first slot in its send order
        N_TRY(ncclGroupStart());
        uint64_t sbase = 0;
        for (uint32_t r = 0; r < P; r++) {
            const uint64_t cnt_in = M[me * P + r];        // my queries served by r
            const uint64_t cnt_out = M[r * P + me];       // r's queries I served
            if (cnt_out)
                N_TRY(ncclSend(d->buf[B_ORES][slot] + seg[r] * 8, cnt_out, ncclUint64, int(r), d->comm, o));
            if (cnt_in) N_TRY(ncclRecv(d->buf[B_RES][slot] + sbase * 8, cnt_in, ncclUint64, int(r), d->comm, o));
            sbase += cnt_in;
        }
        N_TRY(ncclGroupEnd());
    }
    return CUART_OK;
}

// Source role, after the owners: wait for the results (P2P), gather into query order.
cuart_status back(cuart_index* h, DistState* d, const Call& c, uint64_t ci, unsigned long long seq,
                  const unsigned long long* M) {
    (void)h;
    const uint32_t slot = uint32_t(ci & 1);
    const uint64_t b0 = ci * d->chunk;
    const uint64_t m = b0 < c.n ? std::min<uint64_t>(d->chunk, c.n - b0) : 0;
    cudaStream_t s = d->S;
    if (d->transport == CUART_TRANSPORT_P2P) {
        k_wait_flags<<<1, 32, 0, s>>>(d->ctrl, d->P, F_RES, seq);
        g_cuart_launches++;
    }
    if (!c.update && m) {
        const uint64_t tiles = (m + kBucketTile - 1) / kBucketTile;
        if (c.flags) {                                // a mixed batch's lookups: update ops get CUART_MISS
            uint64_t kept = 0;
            for (uint32_t o = 0; o < d->P; o++) kept += M[uint64_t(d->rank) * d->P + o];
            k_bgather<false, true><<<unsigned(tiles), kBucketThreads, 0, s>>>(
                (const uint64_t*)d->buf[B_RES][slot], d->jpos[slot], m, d->hist[slot], d->tot[slot], c.out + b0,
                SegOut{}, kept);
        } else {
            k_bgather<false><<<unsigned(tiles), kBucketThreads, 0, s>>>((const uint64_t*)d->buf[B_RES][slot],
                                                                       d->jpos[slot], m, d->hist[slot], d->tot[slot],
                                                                       c.out + b0);
        }
        g_cuart_launches++;
    }
    D_TRY(cudaGetLastError());
    return CUART_OK;
}

template <class Key>
cuart_status run_call(cuart_index* h, DistState* d, const Call& c) {
    DBG("rank %d call %s n %llu", d->rank, c.update ? "update" : "lookup", (unsigned long long)c.n);
    // agree on the number of chunks: every rank publishes its n (one small round)
    const unsigned long long seq0 = ++d->seq;
    const uint32_t P = d->P;
    uint64_t nmax = c.n;
    if (P > 1) {
        if (d->transport == CUART_TRANSPORT_P2P) {
            // row of n's through the CNT machinery, in its own slot (2)
            const uint32_t slot = 2;
            const Peers pe = peers_of(d);
            k_publish<<<1, 32, 0, d->S>>>(pe, slot, nullptr, c.n, d->lbpo, 1u, seq0);
            k_wait_counts<<<1, 32, 0, d->S>>>(d->ctrl, P, uint32_t(d->rank), slot, seq0, nullptr, d->lbpo, 1u,
                                              d->adj[slot], d->hmat + slot * (size_t(P) * P + 1));
            g_cuart_launches += 2;
            D_TRY(cudaGetLastError());
            cuart_status rc = host_wait_matrix(d, slot, seq0);
            if (rc != CUART_OK) return rc;
            const unsigned long long* M = d->hmat + slot * (size_t(P) * P + 1);
            for (uint32_t s = 0; s < P; s++) nmax = std::max<uint64_t>(nmax, M[s * P]);
        } else {
            unsigned long long mine = c.n;
            D_TRY(cudaMemcpyAsync(d->row, &mine, 8, cudaMemcpyHostToDevice, d->S));
            N_TRY(ncclAllGather(d->row, d->mat, 1, ncclUint64, d->comm, d->S));
            D_TRY(cudaMemcpyAsync(d->hrow, d->mat, size_t(P) * 8, cudaMemcpyDeviceToHost, d->S));
            D_TRY(cudaStreamSynchronize(d->S));
            for (uint32_t s = 0; s < P; s++) nmax = std::max<uint64_t>(nmax, d->hrow[s]);
        }
    }
    const uint64_t nc = (nmax + d->chunk - 1) / d->chunk;
    d->last_recv = 0;
    d->last_chunks = nc;
    if (nc == 0) return CUART_OK;
    const bool p2p = d->transport == CUART_TRANSPORT_P2P;
    const unsigned long long base = d->seq;           // chunk ci uses seq base + 1 + ci
    d->seq += nc;
    if (c.update && nc) {
        // one epoch for every chunk of the call: priorities are global (reading C7)
        cudaStream_t o = p2p ? d->O : d->S;
        cuart_status rc = next_epoch(h, o);
        if (rc != CUART_OK) return rc;
        h->hold_epoch = true;
    }
    cuart_status rc = CUART_OK;
    if (!p2p) {
        for (uint64_t ci = 0; ci < nc && rc == CUART_OK; ci++) {
            rc = front<Key>(h, d, c, ci, base + 1 + ci);
            if (rc == CUART_OK) rc = owner(h, d, c, ci, base + 1 + ci, d->hrow);
            if (rc == CUART_OK) rc = back(h, d, c, ci, base + 1 + ci, d->hrow);
        }
    } else {
        rc = front<Key>(h, d, c, 0, base + 1);
        for (uint64_t ci = 0; ci < nc && rc == CUART_OK; ci++) {
            if (ci + 1 < nc) rc = front<Key>(h, d, c, ci + 1, base + 2 + ci);
            if (rc != CUART_OK) break;
            const uint32_t slot = uint32_t(ci & 1);
            rc = host_wait_matrix(d, slot, base + 1 + ci);
            DBG("rank %d chunk %llu matrix rc %d", d->rank, (unsigned long long)ci, int(rc));
            if (rc != CUART_OK) break;
            rc = owner(h, d, c, ci, base + 1 + ci, d->hmat + slot * (size_t(P) * P + 1));
            if (rc == CUART_OK) rc = back(h, d, c, ci, base + 1 + ci, d->hmat + slot * (size_t(P) * P + 1));
        }
    }
    h->hold_epoch = false;
    return rc;
}

cuart_status dist_call(cuart_index* h, const cuart_keys* k, const uint64_t* vals, uint64_t* out, size_t n, void* stream,
                       bool update, const uint8_t* flags = nullptr) {
    if (!h || !h->dist || !k) return CUART_ERR_INVALID_ARGUMENT;
    DistState* d = h->dist;
    if (d->failed) return CUART_ERR_INTERNAL;
    if (uint32_t(k->kind) != h->key_kind) return CUART_ERR_INVALID_ARGUMENT;
    if (n > 0 && (!k->data || (update ? !vals : !out))) return CUART_ERR_INVALID_ARGUMENT;
    if (n > 0 && k->kind == CUART_KEY_BYTES && !k->lengths) return CUART_ERR_INVALID_ARGUMENT;
    if (uint64_t(n) > (uint64_t(1) << 32) / d->P) return CUART_ERR_INVALID_ARGUMENT;
    D_TRY(cudaSetDevice(h->device));
    cudaStream_t us = (cudaStream_t)stream;
    // internal streams join the caller's stream at entry and it joins them at exit
    D_TRY(cudaEventRecord(d->ev_in, us));
    D_TRY(cudaStreamWaitEvent(d->S, d->ev_in, 0));
    D_TRY(cudaStreamWaitEvent(d->O, d->ev_in, 0));
    if (flags) {                                    // a mixed round: all lookups, then all updates (reading C7)
        if (d->mode != CUART_DIST_RANGE || (n > 0 && (!vals || !out))) return CUART_ERR_INVALID_ARGUMENT;
        Call cl{k->data, k->lengths, nullptr, out, uint64_t(n), false, flags};
        Call cu{k->data, k->lengths, vals, nullptr, uint64_t(n), true, flags};
        cuart_status rc;
        switch (h->key_kind) {
        case CUART_KEY_U64: rc = run_call<KeyU64>(h, d, cl); if (rc == CUART_OK) rc = run_call<KeyU64>(h, d, cu); break;
        case CUART_KEY_U32: rc = run_call<KeyU32>(h, d, cl); if (rc == CUART_OK) rc = run_call<KeyU32>(h, d, cu); break;
        default: rc = run_call<KeyBytes>(h, d, cl); if (rc == CUART_OK) rc = run_call<KeyBytes>(h, d, cu); break;
        }
        if (rc != CUART_OK) d->failed = true;
        D_TRY(cudaEventRecord(d->ev_s, d->S));
        D_TRY(cudaEventRecord(d->ev_o, d->O));
        D_TRY(cudaStreamWaitEvent(us, d->ev_s, 0));
        D_TRY(cudaStreamWaitEvent(us, d->ev_o, 0));
        return rc;
    }
    Call c{k->data, k->lengths, vals, out, uint64_t(n), update};
    if (!update && d->mode == CUART_DIST_REPLICA) {   // replicas: served locally, no exchange
        cuart_status rc = launch_lookup(h, h->key_kind, k->data, k->lengths, n, out, d->S);
        d->last_recv = n;
        d->last_chunks = 0;
        D_TRY(cudaEventRecord(d->ev_s, d->S));
        D_TRY(cudaStreamWaitEvent(us, d->ev_s, 0));
        return rc;
    }
    cuart_status rc;
    switch (h->key_kind) {
    case CUART_KEY_U64: rc = run_call<KeyU64>(h, d, c); break;
    case CUART_KEY_U32: rc = run_call<KeyU32>(h, d, c); break;
    default: rc = run_call<KeyBytes>(h, d, c); break;
    }
    if (rc != CUART_OK) d->failed = true;          // the group's protocol state is unknown now
    D_TRY(cudaEventRecord(d->ev_s, d->S));
    D_TRY(cudaEventRecord(d->ev_o, d->O));
    D_TRY(cudaStreamWaitEvent(us, d->ev_s, 0));
    D_TRY(cudaStreamWaitEvent(us, d->ev_o, 0));
    return rc;
}

cuart_status setup_buffers(cuart_index* h, DistState* d) {
    const uint32_t P = d->P;
    const bool strings = d->kind == CUART_KEY_BYTES;
    const bool p2p = d->transport == CUART_TRANSPORT_P2P;
    const uint64_t C = d->chunk, W = d->wcap;
    void* p = nullptr;
    cuart_status rc;
    if ((rc = dalloc(d, &p, sizeof(Ctrl))) != CUART_OK) return rc;
    d->ctrl = (Ctrl*)p;
    D_TRY(cudaMemset(d->ctrl, 0, sizeof(Ctrl)));
    const size_t bytes[kNumBuf] = {W * d->ks, strings ? W : 0, W * 8, W * 4, C * 8,
                                   p2p ? 0 : C * d->ks, p2p || !strings ? 0 : C, p2p ? 0 : C * 8, p2p ? 0 : C * 4,
                                   p2p ? 0 : W * 8};
    for (int b = 0; b < kNumBuf; b++)
        for (int sl = 0; sl < 2; sl++) {
            if (!bytes[b]) continue;
            if ((rc = dalloc(d, &p, bytes[b])) != CUART_OK) return rc;
            d->buf[b][sl] = (uint8_t*)p;
        }
    const uint64_t tiles = (C + kBucketTile - 1) / kBucketTile;
    for (int sl = 0; sl < 2; sl++) {
        if ((rc = dalloc(d, &p, hist_entries(tiles) * 4)) != CUART_OK) return rc;
        d->hist[sl] = (unsigned int*)p;
        if ((rc = dalloc(d, &p, 2048)) != CUART_OK) return rc;
        d->tot[sl] = (unsigned int*)p;
        if ((rc = dalloc(d, &p, C * 2)) != CUART_OK) return rc;
        d->jpos[sl] = (uint16_t*)p;
    }
    for (int sl = 0; sl < 3; sl++) {
        if ((rc = dalloc(d, &p, kMaxRanks * 8)) != CUART_OK) return rc;
        d->adj[sl] = (long long*)p;
        D_TRY(cudaMemset(d->adj[sl], 0, kMaxRanks * 8));
    }
    if ((rc = dalloc(d, &p, kMaxRanks * 8)) != CUART_OK) return rc;
    d->row = (unsigned long long*)p;
    if ((rc = dalloc(d, &p, kMaxRanks * kMaxRanks * 8)) != CUART_OK) return rc;
    d->mat = (unsigned long long*)p;
    D_TRY(cudaHostAlloc((void**)&d->hmat, 3 * (size_t(P) * P + 1) * 8, cudaHostAllocMapped | cudaHostAllocPortable));
    memset(d->hmat, 0, 3 * (size_t(P) * P + 1) * 8);
    D_TRY(cudaHostAlloc((void**)&d->hrow, kMaxRanks * kMaxRanks * 8, cudaHostAllocPortable));
    // peers: exchange the windows that remote ranks write (P2P): ctrl, receive windows, results
    for (int b = 0; b < kNumBuf; b++)
        for (int sl = 0; sl < 2; sl++) d->peer[b][sl][d->rank] = d->buf[b][sl];
    d->pctrl[d->rank] = d->ctrl;
    if (!p2p || P == 1) return CUART_OK;
    const int exp[] = {B_KEYS, B_LENS, B_VALS, B_PRIO, B_RES};
    const int nexp = 1 + 2 * 5;
    std::vector<WinHandle> mine(nexp), all(size_t(nexp) * P);
    auto fill = [&](WinHandle& w, void* ptr) -> cuart_status {
        memset(&w, 0, sizeof(w));
        w.pid = int(getpid());
        w.dev = h->device;
        w.ptr = ptr;
        if (ptr) {
            cudaIpcMemHandle_t hd;
            D_TRY(cudaIpcGetMemHandle(&hd, ptr));
            memcpy(w.ipc, &hd, sizeof(hd));
        }
        return CUART_OK;
    };
    if ((rc = fill(mine[0], d->ctrl)) != CUART_OK) return rc;
    for (int e = 0; e < 5; e++)
        for (int sl = 0; sl < 2; sl++)
            if ((rc = fill(mine[1 + 2 * e + sl], d->buf[exp[e]][sl])) != CUART_OK) return rc;
    if ((rc = boot_allgather(d, mine.data(), all.data(), sizeof(WinHandle) * nexp)) != CUART_OK) return rc;
    const int me_pid = int(getpid());
    auto open = [&](const WinHandle& w, void** out) -> cuart_status {
        *out = nullptr;
        if (!w.ptr) return CUART_OK;
        if (w.pid == me_pid) {                   // a virtual rank of this process: same address space
            *out = w.ptr;
            return CUART_OK;
        }
        cudaIpcMemHandle_t hd;
        memcpy(&hd, w.ipc, sizeof(hd));
        D_TRY(cudaIpcOpenMemHandle(out, hd, cudaIpcMemLazyEnablePeerAccess));
        d->imported.push_back(*out);
        return CUART_OK;
    };
    for (uint32_t r = 0; r < P; r++) {
        if (r == uint32_t(d->rank)) continue;
        const WinHandle* w = &all[size_t(r) * nexp];
        void* ptr = nullptr;
        if ((rc = open(w[0], &ptr)) != CUART_OK) return rc;
        d->pctrl[r] = (Ctrl*)ptr;
        for (int e = 0; e < 5; e++)
            for (int sl = 0; sl < 2; sl++) {
                if ((rc = open(w[1 + 2 * e + sl], &ptr)) != CUART_OK) return rc;
                d->peer[exp[e]][sl][r] = (uint8_t*)ptr;
            }
    }
    return boot_barrier(d);                      // every rank mapped every window
}

}  // namespace

void dist_teardown(cuart_index* h) {
    DistState* d = h->dist;
    h->dist = nullptr;
    if (!d) return;
    cudaDeviceSynchronize();
    if (d->P > 1) boot_barrier(d);               // no peer still reads / writes our windows
    for (void* p : d->imported) cudaIpcCloseMemHandle(p);
    d->imported.clear();
    if (d->P > 1) boot_barrier(d);               // every peer unmapped ours
    free_state(d);
}

extern "C" {

cuart_status cuart_dist_unique_id(void* id) {
    if (!id) return CUART_ERR_INVALID_ARGUMENT;
    ncclUniqueId u;
    if (ncclGetUniqueId(&u) != ncclSuccess) return CUART_ERR_NCCL;
    static_assert(sizeof(u) == CUART_NCCL_ID_BYTES, "ncclUniqueId size");
    memcpy(id, &u, sizeof(u));
    return CUART_OK;
}

cuart_status cuart_dist_chunk_plan(uint32_t P, uint32_t me, const uint64_t* M, uint64_t* seg_start, uint64_t* res_off,
                                   uint64_t* push_off) {
    if (P == 0 || P > kMaxRanks || me >= P || !M || !seg_start || !res_off || !push_off) return CUART_ERR_INVALID_ARGUMENT;
    chunk_plan(P, me, (const unsigned long long*)M, seg_start, res_off, push_off);
    return CUART_OK;
}

cuart_status cuart_dist_partition(const cuart_dist_cfg* cfg, const cuart_keys* keys, size_t n, uint64_t* splitters,
                                  uint8_t* owner) {
    cuart_status rc = check_cfg(cfg);
    if (rc != CUART_OK) return rc;
    if (!keys || (n > 0 && !keys->data) || (keys->kind == CUART_KEY_BYTES && n > 0 && !keys->lengths))
        return CUART_ERR_INVALID_ARGUMENT;
    if (keys->kind != CUART_KEY_U32 && keys->kind != CUART_KEY_U64 && keys->kind != CUART_KEY_BYTES)
        return CUART_ERR_INVALID_ARGUMENT;
    const uint32_t P = uint32_t(cfg->nranks), kind = uint32_t(keys->kind);
    uint64_t sp[kMaxRanks] = {0};
    if (cfg->mode == CUART_DIST_RANGE && P > 1) {
        if (cfg->splitters) memcpy(sp, cfg->splitters, (P - 1) * 8);
        else if (cfg->keys_local) return CUART_ERR_INVALID_ARGUMENT;
        else quantile_splitters(kind, keys->data, keys->lengths, n, P, sp);
    }
    if (splitters && P > 1) memcpy(splitters, sp, (P - 1) * 8);
    if (owner)
        for (size_t i = 0; i < n; i++)
            owner[i] = cfg->mode == CUART_DIST_RANGE ? uint8_t(owner_host(sp, P - 1, prefix8_host(kind, keys->data, keys->lengths, i)))
                                                     : uint8_t(cfg->rank);
    if (cfg->allgather && P > 1) {                // every rank must hold the same splitters
        std::vector<uint64_t> all(size_t(P) * kMaxRanks);
        if (cfg->allgather(cfg->allgather_ctx, sp, all.data(), kMaxRanks * 8) != 0) return CUART_ERR_NCCL;
        for (uint32_t r = 0; r < P; r++)
            if (memcmp(&all[size_t(r) * kMaxRanks], sp, kMaxRanks * 8) != 0) return CUART_ERR_INVALID_ARGUMENT;
    }
    return CUART_OK;
}

cuart_status cuart_dist_build(const cuart_dist_cfg* cfg, const cuart_keys* keys, const uint64_t* values, size_t n,
                              cuart_index** out) {
    if (!out) return CUART_ERR_INVALID_ARGUMENT;
    *out = nullptr;
    cuart_status rc = check_cfg(cfg);
    if (rc != CUART_OK) return rc;
    if (!keys || (n > 0 && (!keys->data || !values))) return CUART_ERR_INVALID_ARGUMENT;
    if (keys->kind != CUART_KEY_U32 && keys->kind != CUART_KEY_U64 && keys->kind != CUART_KEY_BYTES)
        return CUART_ERR_INVALID_ARGUMENT;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) return CUART_ERR_NO_DEVICE;
    int dev = cfg->opts.device;
    if (dev < 0 && cudaGetDevice(&dev) != cudaSuccess) return CUART_ERR_CUDA;
    if (dev >= ndev) return CUART_ERR_NO_DEVICE;
    if (cudaSetDevice(dev) != cudaSuccess) return CUART_ERR_CUDA;
    const uint32_t P = uint32_t(cfg->nranks), kind = uint32_t(keys->kind);
    DBG("build rank %d/%u mode %u transport %u n %zu dev %d", cfg->rank, P, cfg->mode, cfg->transport, n, dev);
    DistState* d = new (std::nothrow) DistState();
    if (!d) return CUART_ERR_OOM;
    d->rank = cfg->rank;
    d->P = P;
    d->mode = cfg->mode;
    d->transport = cfg->transport;
    d->ag = cfg->allgather;
    d->ag_ctx = cfg->allgather_ctx;
    d->kind = kind;
    d->ks = key_bytes(kind);
    if (cudaStreamCreateWithFlags(&d->S, cudaStreamNonBlocking) != cudaSuccess ||
        cudaStreamCreateWithFlags(&d->O, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&d->ev_in, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&d->ev_o, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&d->ev_s, cudaEventDisableTiming) != cudaSuccess) {
        free_state(d);
        return CUART_ERR_CUDA;
    }
    if (P > 1 && (cfg->transport == CUART_TRANSPORT_NCCL || !cfg->allgather)) {
        ncclUniqueId id;
        memcpy(&id, cfg->nccl_id, sizeof(id));
        if (ncclCommInitRank(&d->comm, int(P), id, cfg->rank) != ncclSuccess) {
            d->comm = nullptr;
            free_state(d);
            return CUART_ERR_NCCL;
        }
    } else if (cfg->transport == CUART_TRANSPORT_NCCL) {   // a 1-rank group still moves data with NCCL calls
        ncclUniqueId id;
        if (ncclGetUniqueId(&id) != ncclSuccess || ncclCommInitRank(&d->comm, 1, id, 0) != ncclSuccess) {
            d->comm = nullptr;
            free_state(d);
            return CUART_ERR_NCCL;
        }
    }
    // partition: splitters (identical on every rank, checked through the bootstrap) and my keys
    uint64_t sp[kMaxRanks] = {0};
    std::vector<uint8_t> own;
    const void* kd = keys->data;
    const uint8_t* kl = keys->lengths;
    const uint64_t* kv = values;
    size_t kn = n;
    std::vector<uint8_t> sel_k, sel_l;
    std::vector<uint64_t> sel_v;
    if (cfg->mode == CUART_DIST_RANGE && P > 1) {
        if (cfg->splitters) memcpy(sp, cfg->splitters, (P - 1) * 8);
        else quantile_splitters(kind, kd, kl, n, P, sp);
        std::vector<uint64_t> all(size_t(P) * kMaxRanks);
        rc = boot_allgather(d, sp, all.data(), kMaxRanks * 8);
        for (uint32_t r = 0; r < P && rc == CUART_OK; r++)
            if (memcmp(&all[size_t(r) * kMaxRanks], sp, kMaxRanks * 8) != 0) rc = CUART_ERR_INVALID_ARGUMENT;
        if (rc != CUART_OK) {
            free_state(d);
            return rc;
        }
        if (!cfg->keys_local) {
            const size_t ks = key_bytes(kind);
            for (size_t i = 0; i < n; i++) {
                if (owner_host(sp, P - 1, prefix8_host(kind, kd, kl, i)) != uint32_t(cfg->rank)) continue;
                sel_k.insert(sel_k.end(), (const uint8_t*)kd + i * ks, (const uint8_t*)kd + (i + 1) * ks);
                if (kl) sel_l.push_back(kl[i]);
                sel_v.push_back(values[i]);
            }
            kd = sel_k.data();
            kl = kl ? sel_l.data() : nullptr;
            kv = sel_v.data();
            kn = sel_v.size();
        }
    }
    DBG("local keys %zu", kn);
    cuart_keys lk{keys->kind, kd, kl};
    cuart_build_opts opts = cfg->opts;
    opts.device = dev;
    cuart_index* h = nullptr;
    rc = cuart_build(&lk, kv, kn, &opts, &h);
    if (rc != CUART_OK) {                            // tell the peers nothing; they fail on the next bootstrap
        free_state(d);
        return rc;
    }
    DBG("local index built");
    h->dist = d;
    for (uint32_t j = 0; j + 1 < P; j++) d->part.sp[j] = sp[j];
    d->part.nsp = cfg->mode == CUART_DIST_RANGE ? P - 1 : 0;
    d->lbpo = P == 1 ? 8 - h->bucket_shift : 8 - ceil_log2(P);
    d->part.lbpo = d->lbpo;
    // every owner's root branch depth (the bucket byte of its parts)
    const uint8_t dep = uint8_t(link_type(h->root) >= T_N4 && link_type(h->root) <= T_N256 ? link_aux(h->root) : 0u);
    std::vector<uint8_t> deps(P);
    if ((rc = boot_allgather(d, &dep, deps.data(), 1)) != CUART_OK) {
        h->dist = nullptr;
        free_state(d);
        cuart_destroy(h);
        return rc;
    }
    for (uint32_t r = 0; r < P; r++) d->part.depth[r] = deps[r];
    // chunk C and window capacity P*C per slot (P*C < 2^32: send-order slots are 32-bit)
    // Default C: the largest power of two whose two window slots (P * C ops of key +
    // length + value + priority each, plus C results) fit a 16 GiB budget
    // (CUART_DIST_WINDOW_BYTES): 2^28 ops at one rank, 2^25 at eight (u64).  Larger
    // chunks walk longer runs of each bucket (more reuse of its tree slice) and pay the
    // per-chunk protocol (a count exchange, ~10 small launches) less often.
    uint64_t budget = uint64_t(16) << 30;
    if (const char* pe = getenv("CUART_DIST_WINDOW_BYTES")) budget = strtoull(pe, nullptr, 0);
    const uint64_t per_op = 2 * (uint64_t(P) * (key_bytes(kind) + (kind == CUART_KEY_BYTES ? 1 : 0) + 12) + 8);
    uint64_t C = uint64_t(1) << 20;
    while (C < (uint64_t(1) << 29) && 2 * C * per_op <= budget) C <<= 1;
    if (cfg->chunk) C = cfg->chunk;
    if (const char* pe = getenv("CUART_DIST_CHUNK")) C = strtoull(pe, nullptr, 0);
    C = std::max<uint64_t>(kBucketTile, (C + kBucketTile - 1) / kBucketTile * kBucketTile);
    while (uint64_t(P) * C >= (uint64_t(1) << 31)) C /= 2;
    d->chunk = C;
    d->wcap = uint64_t(P) * C;
    DBG("chunk %llu window %llu", (unsigned long long)C, (unsigned long long)d->wcap);
    set_scatter_smem<KeyU64, false>();
    set_scatter_smem<KeyU64, true>();
    set_scatter_smem<KeyU32, false>();
    set_scatter_smem<KeyU32, true>();
    set_scatter_smem<KeyBytes, false>();
    set_scatter_smem<KeyBytes, true>();
    rc = setup_buffers(h, d);
    DBG("buffers rc %d", int(rc));
    if (rc != CUART_OK) {
        h->dist = nullptr;
        free_state(d);
        cuart_destroy(h);
        return rc;
    }
    *out = h;
    return CUART_OK;
}

cuart_status cuart_dist_lookup(cuart_index* h, const cuart_keys* q, size_t n, uint64_t* out, void* stream) {
    return dist_call(h, q, nullptr, out, n, stream, false);
}

cuart_status cuart_dist_update(cuart_index* h, const cuart_keys* k, const uint64_t* v, size_t n, void* stream) {
    return dist_call(h, k, v, nullptr, n, stream, true);
}

cuart_status cuart_dist_mixed(cuart_index* h, const cuart_keys* k, const uint64_t* v, const uint8_t* is_update, size_t n,
                              uint64_t* out, void* stream) {
    if (n > 0 && !is_update) return CUART_ERR_INVALID_ARGUMENT;
    static const uint8_t none = 0;
    return dist_call(h, k, v, out, n, stream, false, n ? is_update : &none);
}

cuart_status cuart_dist_last(const cuart_index* h, uint64_t* recv_ops, uint64_t* chunks) {
    if (!h || !h->dist || !recv_ops || !chunks) return CUART_ERR_INVALID_ARGUMENT;
    *recv_ops = h->dist->last_recv;
    *chunks = h->dist->last_chunks;
    return CUART_OK;
}

}  // extern "C"
