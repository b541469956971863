"""Seeded synthetic workload generators shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the method (no key canonicalisation, no tree
logic, no lookup/update semantics): it only draws numbers.  Both the oracle
(``oracle/``) and the product binding consume its arrays; neither imports the
other.  Every draw is a pure function of (stream seed, counter) through the
counter-based splitmix64 mixer, so any element of any stream can be recomputed
on its own (the full-size parity tests sample single elements this way).

Workload recipes follow SURVEY.md §8(d) ("Synthetic inputs") and are restated in
DESIGN.md §"Input recipe".  Key shapes mirror the paper's workloads: random
integer keys ("synthetic random test data"), dense sequential
keys, and variable-length byte strings up to the compile-time maximum of 32 B
(P:110).
"""
from __future__ import annotations

import dataclasses
import numpy as np

MASK64 = (1 << 64) - 1
GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
#: Reserved "absent" value (SURVEY §8(b) CUART_MISS); generated values avoid it.
RESERVED_VALUE = np.uint64(0xFFFFFFFFFFFFFFFF)

# Stream seeds per config c: keys 1000+c, values 1500+c,
# queries 2000+c, updates 3000+c, update values 3500+c.
SEED_KEYS, SEED_VALUES, SEED_QUERIES, SEED_UPDATES, SEED_UVALUES = 1000, 1500, 2000, 3000, 3500


def splitmix64(seed: int, counter) -> np.ndarray:
    """Counter-based splitmix64: mix(seed + (counter+1)*golden).

    For a fixed seed this is a bijection of the counter on [0, 2^64), so draws at
    distinct counters are distinct — used to build key sets with guaranteed
    distinct members and guaranteed-absent miss keys without any membership test.
    """
    c = np.asarray(counter, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = np.uint64(seed & MASK64) + (c + np.uint64(1)) * GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def splitmix64_scalar(seed: int, counter: int) -> int:
    z = (seed + (counter + 1) * 0x9E3779B97F4A7C15) & MASK64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


def values_for(seed: int, counter) -> np.ndarray:
    """u64 payloads, remapped away from the reserved miss value."""
    v = splitmix64(seed, counter)
    v[v == RESERVED_VALUE] = np.uint64(0)
    return v


@dataclasses.dataclass(frozen=True)
class Config:
    name: str
    kind: str              # "u64" | "u32" | "bytes"
    n_keys: int
    n_lookups: int
    n_updates: int
    hit_ratio: float       # fraction of lookups drawn from the key set
    description: str


# BASELINE.json "configs" (sizes read as powers of two where the text says M/B).
CONFIGS = {
    "c1": Config("c1", "u64", 65_536, 1 << 20, 100_000, 0.5,
                 "65,536 random 64-bit keys, 1M point lookups (50% hit) + 100K value updates"),
    "c2": Config("c2", "u32", 1 << 24, 1 << 28, 0, 1.0,
                 "16M dense sequential 32-bit keys, 256M lookups (100% hit)"),
    "c3": Config("c3", "u64", 1 << 26, 1 << 30, 1 << 26, 0.5,
                 "64M sparse uniform-random 64-bit keys, 1B lookups at 50% hit + 64M update batch"),
    "c4": Config("c4", "bytes", 1 << 25, 1 << 29, 0, 1.0,
                 "32M variable-length byte-string keys (8-32 B), 512M Zipf lookups"),
}


def config_id(cfg: Config) -> int:
    return int(cfg.name[1:])


# ----------------------------------------------------------------------------- keys
def u64_keys(c: int, n: int) -> np.ndarray:
    """n distinct uniform-random u64 keys (bijective counter draw, no dedupe needed)."""
    return splitmix64(SEED_KEYS + c, np.arange(n, dtype=np.uint64))


def u64_absent_keys(c: int, n_keys: int, start: int, m: int) -> np.ndarray:
    """m u64 keys guaranteed NOT in u64_keys(c, n_keys): counters >= n_keys of the same bijection."""
    return splitmix64(SEED_KEYS + c, np.arange(n_keys + start, n_keys + start + m, dtype=np.uint64))


def build_set(cfg: Config):
    """(keys, values) for the build call, in generator order (unsorted)."""
    c = config_id(cfg)
    vals = values_for(SEED_VALUES + c, np.arange(cfg.n_keys, dtype=np.uint64))
    if cfg.kind == "u64":
        return u64_keys(c, cfg.n_keys), vals
    if cfg.kind == "u32":
        return np.arange(cfg.n_keys, dtype=np.uint32), vals
    if cfg.kind == "bytes":
        slots, lens = string_keys(c, cfg.n_keys)
        return (slots, lens), vals[: lens.shape[0]]
    raise ValueError(cfg.kind)


def lookup_batch(cfg: Config, keys, start: int = 0, m: int | None = None):
    """Lookup queries [start, start+m) of the config's stream (see lookup_at)."""
    m = cfg.n_lookups - start if m is None else m
    return lookup_at(cfg, keys, np.arange(start, start + m, dtype=np.uint64))


def lookup_at(cfg: Config, keys, j) -> np.ndarray:
    """Lookup queries at absolute stream positions j (any order, any subset).

    u64: query j is a hit (uniform key of the set) when draw 2j < hit_ratio*2^64,
    otherwise a guaranteed-absent key (counter >= n of the key bijection).
    u32 (c2): uniform over [0, 2^24) => 100% hit.
    """
    c = config_id(cfg)
    j = np.asarray(j, dtype=np.uint64)
    m = j.shape[0]
    if cfg.kind == "u32":
        return (splitmix64(SEED_QUERIES + c, j) >> np.uint64(40)).astype(np.uint32)
    if cfg.kind == "u64":
        n = keys.shape[0]
        sel = splitmix64(SEED_QUERIES + c, np.uint64(2) * j)
        pick = splitmix64(SEED_QUERIES + c, np.uint64(2) * j + np.uint64(1))
        if cfg.hit_ratio >= 1.0:
            hit = np.ones(m, dtype=bool)
        else:
            thresh = np.uint64(int(cfg.hit_ratio * 2**64) & MASK64)
            hit = sel < thresh
        out = splitmix64(SEED_KEYS + c, (np.uint64(n) + np.uint64(1 << 40) + j))  # absent: counters >= n
        hk = keys[(pick % np.uint64(n)).astype(np.int64)]
        out[hit] = hk[hit]
        return out
    raise ValueError(cfg.kind)


def update_batch(cfg: Config, keys, start: int = 0, m: int | None = None):
    """Update ops [start, start+m): 90% keys drawn with replacement from the set
    (duplicates exercise last-writer-wins), 10% guaranteed-absent keys."""
    c = config_id(cfg)
    m = cfg.n_updates - start if m is None else m
    j = np.arange(start, start + m, dtype=np.uint64)
    n = keys.shape[0]
    sel = splitmix64(SEED_UPDATES + c, np.uint64(2) * j)
    pick = splitmix64(SEED_UPDATES + c, np.uint64(2) * j + np.uint64(1))
    present = sel < np.uint64(int(0.9 * 2**64))
    if cfg.kind == "u64":
        out = splitmix64(SEED_KEYS + c, (np.uint64(n) + np.uint64(1 << 41) + j))
    elif cfg.kind == "u32":
        out = (np.uint64(n) + j).astype(np.uint32)  # dense set is [0, n): n+j is absent
        keys = keys.astype(np.uint32)
    else:
        raise ValueError(cfg.kind)
    hk = keys[(pick % np.uint64(n)).astype(np.int64)]
    out[present] = hk[present]
    vals = values_for(SEED_UVALUES + c, j)
    return out, vals


# ----------------------------------------------------------------------------- strings
ALPHABET = np.frombuffer(b"abcdefghijklmnopqrstuvwxyz0123456789/.:_-#", dtype=np.uint8)  # 42 symbols
MAX_KEY = 32


def _zipf_index(u01: np.ndarray, n: int, s: float) -> np.ndarray:
    """Inverse-CDF Zipf(s) over ranks [0, n) from uniforms in [0,1)."""
    w = 1.0 / np.arange(1, n + 1, dtype=np.float64) ** s
    cdf = np.cumsum(w)
    cdf /= cdf[-1]
    return np.minimum(np.searchsorted(cdf, u01, side="right"), n - 1)


def _u01(seed: int, counter) -> np.ndarray:
    return (splitmix64(seed, counter) >> np.uint64(11)).astype(np.float64) * (1.0 / (1 << 53))


def string_keys(c: int, n: int, max_len: int = MAX_KEY, min_len: int = 8):
    """n distinct, prefix-free byte-string keys as (slots uint8[n,32], lens uint8[n]).

    Recipe: content = level-1 segment (16 choices, Zipf 1.2) +
    level-2 segment (256 choices, Zipf 1.0), 6 symbols each from a 42-symbol
    alphabet, then random suffix symbols; total length L ~ U{min_len..max_len}
    INCLUDING a 0x00 terminator, so the set is prefix-free (no content byte is 0).
    Duplicates are rejected by drawing extra candidates and keeping the first
    occurrence (order of first appearance is preserved).
    """
    seed = SEED_KEYS + c
    seg1 = ALPHABET[(splitmix64(seed + 11, np.arange(16 * 6, dtype=np.uint64)) % np.uint64(42)).astype(np.int64)].reshape(16, 6)
    seg2 = ALPHABET[(splitmix64(seed + 12, np.arange(256 * 6, dtype=np.uint64)) % np.uint64(42)).astype(np.int64)].reshape(256, 6)
    out_slots, out_lens, out_hash = [], [], []
    have, base = 0, 0
    while have < n:
        m = int((n - have) * 1.35) + 1024
        j = np.arange(base, base + m, dtype=np.uint64)
        base += m
        L = (min_len + (splitmix64(seed + 1, j) % np.uint64(max_len - min_len + 1))).astype(np.int64)
        i1 = _zipf_index(_u01(seed + 2, j), 16, 1.2)
        i2 = _zipf_index(_u01(seed + 3, j), 256, 1.0)
        slots = np.zeros((m, max_len), dtype=np.uint8)
        slots[:, 0:6] = seg1[i1]
        slots[:, 6:12] = seg2[i2]
        for k, col in enumerate(range(12, max_len, 8)):       # 8 suffix symbols per draw
            r = splitmix64(seed + 100 + k, j).view(np.uint8).reshape(m, 8)
            width = min(8, max_len - col)
            slots[:, col: col + width] = ALPHABET[(r[:, :width].astype(np.uint16) * 42) >> 8]
        slots[np.arange(max_len)[None, :] >= (L - 1)[:, None]] = 0          # terminator + zero pad
        # dedupe on a 64-bit digest of the slot (first occurrence wins, draw order kept);
        # a digest collision between distinct keys only drops a candidate
        w = slots.view(np.uint64)
        h = splitmix64(int(w[0, 0]) & 0, w[:, 0])
        for k in range(1, max_len // 8):
            h = splitmix64(0, h ^ w[:, k])
        out_slots.append(slots)
        out_lens.append(L.astype(np.uint8))
        out_hash.append(h)
        allh = np.concatenate(out_hash)
        _, first = np.unique(allh, return_index=True)
        first.sort()
        allslots = np.concatenate(out_slots)[first]
        out_slots, out_lens, out_hash = [allslots], [np.concatenate(out_lens)[first]], [allh[first]]
        have = first.shape[0]
    return out_slots[0][:n].copy(), out_lens[0][:n].copy()


def zipf_ranks(seed: int, counter, n: int, theta: float = 0.99) -> np.ndarray:
    """Zipf(theta) ranks in [0, n) by inverse CDF of counter-based uniforms."""
    w = 1.0 / np.arange(1, n + 1, dtype=np.float64) ** theta
    cdf = np.cumsum(w)
    cdf /= cdf[-1]
    return np.minimum(np.searchsorted(cdf, _u01(seed, counter), side="right"), n - 1)


def rank_permutation(seed: int, n: int) -> np.ndarray:
    """Seeded permutation mapping Zipf rank -> key index (hot keys spread over the set)."""
    return np.argsort(splitmix64(seed, np.arange(n, dtype=np.uint64)), kind="stable")


def string_lookup_at(cfg: Config, n_keys: int, j) -> np.ndarray:
    """Key indices of c4 lookups at stream positions j: Zipf(0.99) over key ranks,
    ranks mapped to keys by a seeded permutation (100% hit)."""
    c = config_id(cfg)
    perm = rank_permutation(SEED_QUERIES + c + 7, n_keys)
    return perm[zipf_ranks(SEED_QUERIES + c, np.asarray(j, dtype=np.uint64), n_keys)]


# ----------------------------------------------------------------------------- torch twins
# The same counter-based draws on torch tensors (CPU or CUDA), for generating the
# full-size batches where they are consumed (device memory) without a host round
# trip.  int64 arithmetic wraps modulo 2^64 exactly like uint64; logical right
# shifts are emulated with a mask.  tests/test_workloads.py pins these to the
# numpy versions bit for bit.
def _t_srl(x, k):
    import torch
    return (x >> k) & ((1 << (64 - k)) - 1)


def _t_const(v):
    return v - (1 << 64) if v >= 1 << 63 else v


def splitmix64_torch(seed: int, counter):
    """torch int64 tensor of splitmix64(seed, counter) bit patterns."""
    z = counter + 1
    z = z * _t_const(0x9E3779B97F4A7C15) + _t_const(seed & MASK64)
    z = (z ^ _t_srl(z, 30)) * _t_const(0xBF58476D1CE4E5B9)
    z = (z ^ _t_srl(z, 27)) * _t_const(0x94D049BB133111EB)
    return z ^ _t_srl(z, 31)


def _t_ult(a, b_const: int):
    """unsigned a < b for int64 bit patterns (b a Python int in [0, 2^64))."""
    import torch
    return (a ^ (-(1 << 63))) < _t_const(b_const ^ (1 << 63))


def _t_umod(a, n: int):
    """unsigned a mod n (n < 2^62) for int64 bit patterns."""
    hi = _t_srl(a, 32)
    lo = a & 0xFFFFFFFF
    return (((hi % n) * ((1 << 32) % n)) % n + lo % n) % n


def u64_keys_torch(c: int, n: int, device):
    import torch
    return splitmix64_torch(SEED_KEYS + c, torch.arange(n, dtype=torch.int64, device=device))


def lookup_batch_torch(cfg: Config, keys, start: int = 0, m: int | None = None, device=None):
    """torch twin of lookup_batch (u64 / u32 configs); returns int64 (u64) or int32 (u32) bits."""
    import torch
    c = config_id(cfg)
    m = cfg.n_lookups - start if m is None else m
    device = keys.device if device is None else device
    j = torch.arange(start, start + m, dtype=torch.int64, device=device)
    if cfg.kind == "u32":
        return _t_srl(splitmix64_torch(SEED_QUERIES + c, j), 40).to(torch.int32)
    n = keys.shape[0]
    sel = splitmix64_torch(SEED_QUERIES + c, 2 * j)
    pick = splitmix64_torch(SEED_QUERIES + c, 2 * j + 1)
    del j
    if cfg.hit_ratio >= 1.0:
        hit = torch.ones(m, dtype=torch.bool, device=device)
    else:
        hit = _t_ult(sel, int(cfg.hit_ratio * 2**64) & MASK64)
    del sel
    out = splitmix64_torch(SEED_KEYS + c, torch.arange(start, start + m, dtype=torch.int64, device=device) + (n + (1 << 40)))
    hk = keys[_t_umod(pick, n)]
    del pick
    return torch.where(hit, hk, out)


def update_batch_torch(cfg: Config, keys, start: int = 0, m: int | None = None):
    import torch
    c = config_id(cfg)
    m = cfg.n_updates - start if m is None else m
    device = keys.device
    j = torch.arange(start, start + m, dtype=torch.int64, device=device)
    n = keys.shape[0]
    sel = splitmix64_torch(SEED_UPDATES + c, 2 * j)
    pick = splitmix64_torch(SEED_UPDATES + c, 2 * j + 1)
    present = _t_ult(sel, int(0.9 * 2**64))
    if cfg.kind != "u64":
        raise ValueError(cfg.kind)
    out = splitmix64_torch(SEED_KEYS + c, j + (n + (1 << 41)))
    out = torch.where(present, keys[_t_umod(pick, n)], out)
    vals = splitmix64_torch(SEED_UVALUES + c, j)
    vals = torch.where(vals == -1, torch.zeros_like(vals), vals)
    return out, vals


def string_lookup_index_torch(cfg: Config, n: int, start: int, m: int, device, cdf_d=None, perm_d=None):
    """torch twin of string_lookup_at for positions [start, start+m): the KEY INDICES
    (int64[m]) the Zipf draws select.  The Zipf CDF is built on the host (numpy,
    exact) and the permutation sorts the same splitmix64 draws as unsigned, so ranks
    and keys match the numpy twin."""
    import torch
    c = config_id(cfg)
    if cdf_d is None:
        w = 1.0 / np.arange(1, n + 1, dtype=np.float64) ** 0.99
        cdf = np.cumsum(w)
        cdf /= cdf[-1]
        cdf_d = torch.from_numpy(cdf).to(device)
    if perm_d is None:
        draws = splitmix64_torch(SEED_QUERIES + c + 7, torch.arange(n, dtype=torch.int64, device=device))
        perm_d = torch.argsort(draws ^ (-(1 << 63)), stable=True)        # unsigned order
    j = torch.arange(start, start + m, dtype=torch.int64, device=device)
    u = _t_srl(splitmix64_torch(SEED_QUERIES + c, j), 11).to(torch.float64) * (1.0 / (1 << 53))
    r = torch.clamp(torch.searchsorted(cdf_d, u, right=True), max=n - 1)
    return perm_d[r]


def string_lookup_torch(cfg: Config, slots_d, lens_d, start: int, m: int, cdf_d=None, perm_d=None):
    """torch twin of string_lookup_at for positions [start, start+m): returns
    (query slots uint8[m,32], lens uint8[m]) gathered on the keys' device."""
    idx = string_lookup_index_torch(cfg, slots_d.shape[0], start, m, slots_d.device, cdf_d, perm_d)
    return slots_d[idx], lens_d[idx]


def zipf_cdf_torch(n: int, device, theta: float = 0.99):
    """The Zipf(theta) CDF over [0, n) (numpy, exact) on `device`, for reuse across chunks."""
    import torch
    w = 1.0 / np.arange(1, n + 1, dtype=np.float64) ** theta
    cdf = np.cumsum(w)
    cdf /= cdf[-1]
    return torch.from_numpy(cdf).to(device)


def rank_permutation_torch(cfg: Config, n: int, device):
    import torch
    draws = splitmix64_torch(SEED_QUERIES + config_id(cfg) + 7, torch.arange(n, dtype=torch.int64, device=device))
    return torch.argsort(draws ^ (-(1 << 63)), stable=True)


def values_torch(seed: int, start: int, m: int, device):
    """torch twin of values_for over counters [start, start+m)."""
    import torch
    v = splitmix64_torch(seed, torch.arange(start, start + m, dtype=torch.int64, device=device))
    return torch.where(v == -1, torch.zeros_like(v), v)


# ----------------------------------------------------------------------------- config 5 (mixed)
# uniform random u64 keys, one global stream of mixed ops: each op
# is an update with p = 0.1 (key drawn from the set), else a lookup (50% hit).
# The stream is cut into rounds of C5_ROUND global ops; rank r of P originates the
# r-th contiguous 1/P slice of every round (reading C7).
C5 = Config("c5", "u64", 1 << 30, 4 << 30, 0, 0.5,
            "1B random 64-bit keys range-partitioned by leading bytes, 4B mixed lookup/update ops (90/10) in rounds")
C5_ROUND = 1 << 29
C5_UPDATE_P = 0.1


def mixed_ops(c: int, n_keys: int, j):
    """numpy: (keys u64, is_update u8, values u64) of global ops at positions j."""
    j = np.asarray(j, dtype=np.uint64)
    upd = splitmix64(SEED_UPDATES + c, np.uint64(3) * j) < np.uint64(int(C5_UPDATE_P * 2**64))
    pick = splitmix64(SEED_UPDATES + c, np.uint64(3) * j + np.uint64(1)) % np.uint64(n_keys)
    hit = splitmix64(SEED_QUERIES + c, np.uint64(2) * j) < np.uint64(1 << 63)
    present = splitmix64(SEED_KEYS + c, pick)                       # keys are a bijection of their index
    absent = splitmix64(SEED_KEYS + c, np.uint64(n_keys) + np.uint64(1 << 40) + j)
    keys = np.where(upd | hit, present, absent)
    vals = values_for(SEED_UVALUES + c, j)
    return keys, upd.astype(np.uint8), vals


def mixed_ops_torch(c: int, n_keys: int, start: int, m: int, device):
    import torch
    j = torch.arange(start, start + m, dtype=torch.int64, device=device)
    upd = _t_ult(splitmix64_torch(SEED_UPDATES + c, 3 * j), int(C5_UPDATE_P * 2**64))
    pick = _t_umod(splitmix64_torch(SEED_UPDATES + c, 3 * j + 1), n_keys)
    hit = _t_ult(splitmix64_torch(SEED_QUERIES + c, 2 * j), 1 << 63)
    present = splitmix64_torch(SEED_KEYS + c, pick)
    absent = splitmix64_torch(SEED_KEYS + c, j + (n_keys + (1 << 40)))
    keys = torch.where(upd | hit, present, absent)
    vals = splitmix64_torch(SEED_UVALUES + c, j)
    vals = torch.where(vals == -1, torch.zeros_like(vals), vals)
    return keys, upd.to(torch.uint8), vals
