"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, bit-exact.

All results are integers (u64 values / CUART_MISS), so the bar is element-wise
equality.  Small configs are compared element by element with the pointer-ART
oracle; full-size configs are compared on sampled outputs with the plain-map
oracle and on properties that hold at any size.
"""
import random

import numpy as np
import pytest
import torch

import paper_conf_icpp_koppehelggp21_b200 as C
import workloads as W
from oracle import ArtOracle, MapOracle, OART_MISS
from tests.artspec import golden_key, load_golden
from tests.layout_decode import to_records

pytestmark = pytest.mark.gpu
MISS = int(OART_MISS)
DEV = "cuda:0"


def _t(a):
    """numpy -> CUDA tensor with the same bits (uint64 -> int64 view)."""
    if isinstance(a, tuple):
        return (_t(a[0]), _t(a[1]))
    if a.dtype == np.uint64:
        return torch.from_numpy(a.view(np.int64)).to(DEV)
    if a.dtype == np.uint32:
        return torch.from_numpy(a.view(np.int32)).to(DEV)
    return torch.from_numpy(a).to(DEV)


def _u64(t):
    return t.cpu().numpy().view(np.uint64)


def _strings(keys):
    slots = np.zeros((len(keys), 32), np.uint8)
    lens = np.zeros(len(keys), np.uint8)
    for i, k in enumerate(keys):
        slots[i, : len(k)] = np.frombuffer(k, np.uint8)
        lens[i] = len(k)
    return slots, lens


def _as_input(kind, keys):
    if kind == "u64":
        return np.array([int.from_bytes(k, "big") for k in keys], np.uint64)
    if kind == "u32":
        return np.array([int.from_bytes(k, "big") for k in keys], np.uint32)
    return _strings(keys)


def _lookup(ix, q):
    qt = _t(q)
    n = (qt[0] if isinstance(qt, tuple) else qt).shape[0]
    out = torch.empty(n, dtype=torch.int64, device=DEV)
    ix.lookup(qt, out)
    torch.cuda.synchronize()
    return _u64(out)


@pytest.mark.parametrize("name", ["ex_a_u64.json", "ex_d_strings.json", "ex_e_prefix_split.json", "ex_f_long_prefix.json"])
@pytest.mark.parametrize("lut", [0, 1, 3])
def test_golden_gpu(name, lut):
    g = load_golden(name)
    kind = g["kind"]
    inp = _as_input(kind, [golden_key(kind, k) for k in g["keys"]])
    ix = C.Index(inp, np.array(g["values"], np.uint64), lut_bytes=lut)
    qs = [golden_key(kind, q) for q, _ in g["lookups"]]
    exp = [MISS if v is None else v for _, v in g["lookups"]]
    assert _lookup(ix, _as_input(kind, qs) if kind != "bytes" else _strings(qs)).tolist() == exp
    uk = [golden_key(kind, k) for k, _ in g["update_ops"]]
    ix.update(_t(_as_input(kind, uk) if kind != "bytes" else _strings(uk)),
              _t(np.array([v for _, v in g["update_ops"]], np.uint64)))
    ak = [golden_key(kind, k) for k, _ in g["after_update"]]
    got = _lookup(ix, _as_input(kind, ak) if kind != "bytes" else _strings(ak)).tolist()
    assert got == [v for _, v in g["after_update"]]
    ix.close()


@pytest.mark.parametrize("lut,fmt", [(0, 1), (2, 1), (3, 1), (3, 2), (3, 3), (2, 3)])
def test_c1_full_parity(lut, fmt):
    """Config 1 at full size, element by element against the pointer-ART oracle:
    1M lookups (50% hit), 100K updates, then the post-update dump."""
    cfg = W.CONFIGS["c1"]
    keys, vals = W.build_set(cfg)
    o = ArtOracle(keys, vals)
    ix = C.Index(keys, vals, lut_bytes=lut, lut_format=fmt)
    st = ix.stats()
    assert lut == 0 or st["lut_format"] == fmt
    os_ = o.stats()
    assert (st["n4"], st["n16"], st["n48"], st["n256"], st["leaf8"]) == (os_["n4"], os_["n16"], os_["n48"], os_["n256"], os_["leaves"])
    q = W.lookup_batch(cfg, keys)
    got = _lookup(ix, q)
    exp = o.lookup(q)
    assert np.array_equal(got, exp)
    assert abs((exp != OART_MISS).mean() - 0.5) < 0.01
    uk, uv = W.update_batch(cfg, keys)
    ix.update(_t(uk), _t(uv))
    o.update(uk, uv)
    torch.cuda.synchronize()
    assert ix.get_error() == 0
    assert np.array_equal(_lookup(ix, keys), o.lookup(keys))
    assert np.array_equal(_lookup(ix, q), o.lookup(q))
    # full post-update tree state: device dump decoded == oracle structure (incl. values)
    assert to_records(ix.dump()) == o.dump_structure().tolist()
    ix.close()


@pytest.mark.parametrize("mode", ["u64", "u64_shared", "u32", "bytes"])
@pytest.mark.parametrize("seed", range(3))
def test_random_sets_gpu(mode, seed):
    rng = random.Random(seed * 7 + len(mode))
    n = rng.choice([1, 2, 5, 17, 49, 257, 5000, 40_000])
    s = set()
    while len(s) < n:
        if mode == "u64":
            s.add(rng.getrandbits(64).to_bytes(8, "big"))
        elif mode == "u64_shared":
            k = bytearray(8)
            for i in range(rng.randrange(0, 8), 8):
                k[i] = rng.choice([0, 0xFF, rng.randrange(256), rng.randrange(3)])
            s.add(bytes(k))
        elif mode == "u32":
            s.add(rng.choice([rng.getrandbits(32), rng.getrandbits(14)]).to_bytes(4, "big"))
        else:
            stem = rng.choice([b"", b"a", b"q" * 14, b"r" * 15, b"s" * 16, b"t" * 24])
            body = bytes(rng.choice(b"abz\x01\xff") for _ in range(rng.randrange(0, 31 - len(stem) + 1)))
            s.add((stem + body)[:31] + b"\x00")
    keys = sorted(s)
    rng.shuffle(keys)
    kind = "bytes" if mode == "bytes" else ("u32" if mode == "u32" else "u64")
    vals = np.array([rng.getrandbits(63) for _ in keys], np.uint64)
    inp = _as_input(kind, keys)
    o = ArtOracle(inp, vals)
    probes = list(keys)
    for k in keys[:2000]:
        f = bytearray(k)
        f[rng.randrange(len(k))] ^= 1 << rng.randrange(8)
        probes.append(bytes(f))
        if kind == "bytes":
            probes += [k[:-1] or b"\x01", k + b"\x01" if len(k) < 32 else k]
    if kind != "bytes":
        L = 8 if kind == "u64" else 4
        probes = [p for p in probes if len(p) == L] + [rng.getrandbits(8 * L).to_bytes(L, "big") for _ in range(999)]
    pin = _as_input(kind, probes)
    exp = o.lookup(pin)
    for lut, fmt in ((0, 1), (1, 3), (2, 1), (2, 2), (2, 3), (3, 1), (3, 2), (3, 3)):
        ix = C.Index(inp, vals, lut_bytes=lut, lut_format=fmt)
        assert np.array_equal(_lookup(ix, pin), exp), (lut, fmt)
        assert to_records(ix.dump()) == o.dump_structure().tolist()
        ix.close()
    # updates with heavy duplication (last writer wins) + absent keys
    ix = C.Index(inp, vals, lut_bytes=2, lut_format=3)
    m = 3 * len(probes)
    pick = [rng.randrange(len(probes)) for _ in range(m)]
    ukeys = [probes[i] for i in pick]
    uvals = np.array([rng.getrandbits(63) for _ in range(m)], np.uint64)
    uin = _as_input(kind, ukeys)
    ix.update(_t(uin), _t(uvals))
    o.update(uin, uvals)
    assert np.array_equal(_lookup(ix, pin), o.lookup(pin))
    assert to_records(ix.dump()) == o.dump_structure().tolist()
    ix.close()


def test_edge_cases():
    # empty index: everything misses; n = 0 calls are no-ops
    ix = C.Index(np.zeros(0, np.uint64), np.zeros(0, np.uint64), lut_bytes=0)
    assert _lookup(ix, np.array([0, 1, 2**63], np.uint64)).tolist() == [MISS] * 3
    ix.lookup(_t(np.zeros(0, np.uint64)), torch.empty(0, dtype=torch.int64, device=DEV))
    ix.update(_t(np.zeros(0, np.uint64)), _t(np.zeros(0, np.uint64)))
    ix.close()
    # single key: root is a leaf
    ix = C.Index(np.array([42], np.uint64), np.array([7], np.uint64), lut_bytes=3)
    assert _lookup(ix, np.array([42, 43, 0], np.uint64)).tolist() == [7, MISS, MISS]
    ix.close()
    # ragged batch sizes around the CTA size
    cfg = W.CONFIGS["c1"]
    keys, vals = W.build_set(cfg)
    ix = C.Index(keys, vals)
    mp = MapOracle(keys, vals)
    for m in (1, 255, 256, 257, 1000, 65_537):
        q = W.lookup_batch(cfg, keys, 11, m)
        assert np.array_equal(_lookup(ix, q), mp.lookup(q))
    ix.close()


@pytest.mark.parametrize("prebucket", [1, 2])
def test_reserved_value_update_sets_sticky_error(prebucket):
    """Reading C5: an op carrying CUART_MISS is dropped and sets the sticky flag;
    the post-batch state equals the oracle's (which drops the same ops)."""
    keys = np.array([1, 2, 3], np.uint64)
    ix = C.Index(keys, np.array([10, 20, 30], np.uint64), prebucket=prebucket)
    o = ArtOracle(keys, np.array([10, 20, 30], np.uint64))
    for uk, uv in ((np.array([1, 2], np.uint64), np.array([MISS, 5], np.uint64)),
                   (np.array([3, 3, 2], np.uint64), np.array([7, MISS, MISS], np.uint64))):
        ix.update(_t(uk), _t(uv))
        torch.cuda.synchronize()
        o.update(uk, uv)
        assert o.last_rejected > 0
        assert ix.get_error() == 4
        assert ix.get_error() == 0                       # cleared on read
        assert _lookup(ix, keys).tolist() == o.lookup(keys).tolist()
    ix.close()
    # a large batch with reserved values sprinkled in, through the bucketed path
    cfg = W.CONFIGS["c1"]
    keys, vals = W.build_set(cfg)
    ix = C.Index(keys, vals, lut_bytes=3, prebucket=prebucket)
    o = MapOracle(keys, vals)
    uk, uv = W.update_batch(cfg, keys)
    uv = uv.copy()
    uv[::97] = OART_MISS
    ix.update(_t(uk), _t(uv))
    torch.cuda.synchronize()
    o.update(uk, uv)
    assert ix.get_error() == 4
    assert np.array_equal(_lookup(ix, keys), o.lookup(keys))
    ix.close()


def test_host_buffer_paths_match_device():
    cfg = W.CONFIGS["c1"]
    keys, vals = W.build_set(cfg)
    ix = C.Index(keys, vals, lut_bytes=3)
    mp = MapOracle(keys, vals)
    q = W.lookup_batch(cfg, keys)
    assert np.array_equal(ix.lookup_host(q), mp.lookup(q))
    uk, uv = W.update_batch(cfg, keys)
    ix.update_host(uk, uv)
    mp.update(uk, uv)
    assert np.array_equal(ix.lookup_host(keys), mp.lookup(keys))
    ix.close()


@pytest.mark.parametrize("kind", ["u64", "bytes"])
def test_host_pipeline_many_chunks(kind, monkeypatch):
    """cuart_lookup_host / cuart_update_host with 4096-op chunks (CUART_STAGE_CHUNK,
    read when the handle's staging buffers are allocated): lookups spread over the 4
    staging streams, update chunks whose H2D copies overlap the previous chunks'
    kernels while the kernels stay in op order — duplicates across chunks must
    still resolve to the last op, exactly as the plain map."""
    monkeypatch.setenv("CUART_STAGE_CHUNK", "4096")
    rng = np.random.default_rng(21)
    if kind == "u64":
        keys, vals = W.build_set(W.CONFIGS["c1"])
    else:
        keys = W.string_keys(4, 1 << 14)
        vals = np.arange(1 << 14, dtype=np.uint64) + 3
    n = keys[1].shape[0] if isinstance(keys, tuple) else keys.shape[0]
    ix = C.Index(keys, vals, lut_bytes=0 if kind == "bytes" else 3)
    mp = MapOracle(keys, vals)
    pick = rng.integers(0, min(n, 500), 60_001)                    # many duplicates, across chunks
    uk = (keys[0][pick].copy(), keys[1][pick].copy()) if isinstance(keys, tuple) else keys[pick].copy()
    uv = rng.integers(0, 2**63, pick.shape[0], dtype=np.uint64)
    ix.update_host(uk, uv)
    mp.update(uk, uv)
    assert np.array_equal(ix.lookup_host(keys), mp.lookup(keys))
    ix.close()


@pytest.mark.parametrize("form,tg", [("tile", None), ("tile", "1"), ("tile", "33"), ("tile", "64"), ("global", None)])
@pytest.mark.parametrize("shift", ["0", "2", "3"])
def test_prebucket_bucket_counts_and_skew(shift, form, tg, monkeypatch):
    """K-BUCKET with 256 / 64 / 32 buckets (CUART_BUCKET_SHIFT, read at upload) on
    skewed batches: every query in one bucket, queries in two buckets, and a ragged
    uniform batch; lookups and a bucketed update batch must equal the plain map.
    Both batch forms; the tile form also with 1 and 32 tiles per walk CTA
    (CUART_TILE_GROUP) and 33 / 64 (the run table spans both scanning warps)."""
    monkeypatch.setenv("CUART_BUCKET_SHIFT", shift)
    if tg:
        monkeypatch.setenv("CUART_TILE_GROUP", tg)
    rng = np.random.default_rng(int(shift) + 40)
    keys, vals = W.build_set(W.CONFIGS["c1"])
    ix = C.Index(keys, vals, lut_bytes=3, prebucket=C.PREBUCKET_ON, wide_lut=C.WIDE_ON,
                 bucket_form=C.BUCKET_TILE if form == "tile" else C.BUCKET_GLOBAL)
    mp = MapOracle(keys, vals)
    top = keys >> np.uint64(56)
    one = keys[top == top[0]]
    two = keys[(top == top[0]) | (top == top[1])]
    batches = [one[rng.integers(0, one.shape[0], 20_000)],
               np.concatenate([two[rng.integers(0, two.shape[0], 9_000)],
                               (rng.integers(0, 2**56, 3_000, dtype=np.uint64) | (top[0] << np.uint64(56)))]),
               np.where(rng.random(70_001) < 0.5, keys[rng.integers(0, keys.shape[0], 70_001)],
                        rng.integers(0, 2**64, 70_001, dtype=np.uint64))]
    for q in batches:
        assert np.array_equal(_lookup(ix, q), mp.lookup(q))
    uk = one[rng.integers(0, one.shape[0], 30_000)]
    uv = rng.integers(0, 2**63, uk.shape[0], dtype=np.uint64)
    ix.update(_t(uk), _t(uv))
    mp.update(uk, uv)
    assert np.array_equal(_lookup(ix, keys), mp.lookup(keys))
    ix.close()


@pytest.mark.parametrize("n", [4096, 70_001, 3 * 4096 + 1])
def test_prebucket_gather_misaligned_out(n):
    """The pre-bucketed lookup's final gather writes a caller-owned `out` of any
    8-B alignment: an `out` view 8 B into its buffer, and an aligned one, both
    equal the plain map (ragged and odd tile tails included) and nothing outside
    the view is written."""
    rng = np.random.default_rng(n)
    keys, vals = W.build_set(W.CONFIGS["c1"])
    ix = C.Index(keys, vals, lut_bytes=3, prebucket=C.PREBUCKET_ON, wide_lut=C.WIDE_ON)
    mp = MapOracle(keys, vals)
    q = np.where(rng.random(n) < 0.5, keys[rng.integers(0, keys.shape[0], n)],
                 rng.integers(0, 2**64, n, dtype=np.uint64))
    want = mp.lookup(q)
    for off in (0, 1):
        buf = torch.full((n + 2,), 7, dtype=torch.int64, device=DEV)
        out = buf[off:off + n]
        ix.lookup(_t(q), out)
        torch.cuda.synchronize()
        got = buf.cpu().numpy().view(np.uint64)
        assert np.array_equal(got[off:off + n], want)
        assert got[off + n] == 7 and (off == 0 or got[0] == 7)
    ix.close()


@pytest.mark.parametrize("kind", ["u64", "u32"])
def test_prebucket_misaligned_queries(kind):
    """The tile sort loads keys in 16-B vectors only from a 16-B-aligned batch; a
    query view 4 / 8 B into its buffer takes the strided 8-B path.  Both equal the
    plain map, with a ragged tail tile."""
    rng = np.random.default_rng(77)
    if kind == "u64":
        keys, vals = W.build_set(W.CONFIGS["c1"])
        q = np.where(rng.random(70_003) < 0.5, keys[rng.integers(0, keys.shape[0], 70_003)],
                     rng.integers(0, 2**64, 70_003, dtype=np.uint64))
        tdt = torch.int64
    else:
        keys = np.unique((np.arange(1 << 17, dtype=np.uint32) * 29) & np.uint32(0xFFFFFF))
        vals = np.arange(keys.shape[0], dtype=np.uint64) + 1
        q = rng.integers(0, 1 << 24, 70_003, dtype=np.uint32)
        tdt = torch.int32
    ix = C.Index(keys, vals, lut_bytes=3, prebucket=C.PREBUCKET_ON, wide_lut=C.WIDE_ON)
    mp = MapOracle(keys, vals)
    want = mp.lookup(q)
    for off in (0, 1):
        buf = torch.zeros(q.shape[0] + 1, dtype=tdt, device=DEV)
        qv = buf[off:off + q.shape[0]]
        qv.copy_(torch.from_numpy(q.view(np.int64 if kind == "u64" else np.int32)).to(DEV))
        out = torch.empty(q.shape[0], dtype=torch.int64, device=DEV)
        ix.lookup(qv, out)
        torch.cuda.synchronize()
        assert np.array_equal(out.cpu().numpy().view(np.uint64), want), off
    ix.close()


def test_c2_full_size_sampled():
    """Config 2 at full size (2^24 dense u32 keys, LUT over the first 3 bytes):
    2^28 lookups in the bench's launch configuration; sampled outputs vs the
    plain map, and the any-size property out[i] == value(q[i]) (100% hit)."""
    cfg = W.CONFIGS["c2"]
    keys, vals = W.build_set(cfg)
    ix = C.Index(keys, vals, lut_bytes=3, lut_format=3)
    st = ix.stats()
    assert st["n256"] == 1 + 256 + 65_536 and st["leaf8"] == 1 << 24   # Ex-C closed form
    assert st["lut_format"] == 3 and st["lut_exceptions"] == 0
    qd = W.lookup_batch_torch(cfg, torch.zeros(1, dtype=torch.int64, device=DEV), 0, cfg.n_lookups, device=DEV)
    out = torch.empty(cfg.n_lookups, dtype=torch.int64, device=DEV)
    ix.lookup(qd, out)
    torch.cuda.synchronize()
    # property at full size: value table gathered by key (dense keys: value index = key)
    vt = torch.from_numpy(vals.view(np.int64)).to(DEV)
    assert torch.equal(out, vt[qd.long()])
    # sampled, element by element vs the plain-map oracle
    idx = np.sort(np.random.default_rng(5).choice(cfg.n_lookups, 200_000, replace=False))
    qs = W.lookup_at(cfg, None, idx)
    assert np.array_equal(qd[torch.from_numpy(idx).to(DEV)].cpu().numpy().view(np.uint32), qs)
    mp = MapOracle(keys, vals)
    assert np.array_equal(_u64(out[torch.from_numpy(idx).to(DEV)]), mp.lookup(qs))
    ix.close()


@pytest.mark.slow
def test_c3_full_size_every_lookup_and_post_update_state():
    """Config 3 at full size in the bench's launch configuration (2^26 random u64
    keys, one 2^30-query lookup call, one 2^26-op update call):

    * EVERY lookup against its closed form from the generator (plain definition
      M[q]: a hit query is key #pick of the set, whose value is vals[pick]; a miss
      query is a guaranteed-absent key -> CUART_MISS), cross-checked against the
      plain-map oracle on a 300K sample (pins the closed form to the oracle);
    * the FULL post-update tree state: every one of the 2^26 keys looked
      up against the plain-map oracle's sequential replay of the batch, and the
      device dump compared with the pre-update dump -- inner-node buffers and root
      table byte-identical (updates are non-structural), leaf keys unchanged and
      leaf values equal to the oracle's values in key order (leaves are stored in
      lexicographic order)."""
    cfg = W.CONFIGS["c3"]
    n = cfg.n_keys
    keys_d = W.u64_keys_torch(3, n, DEV)
    keys = _u64(keys_d)
    vals = W.values_for(W.SEED_VALUES + 3, np.arange(n, dtype=np.uint64))
    ix = C.Index(keys, vals, lut_bytes=3)
    pre = ix.dump()
    nl = cfg.n_lookups
    out = torch.empty(nl, dtype=torch.int64, device=DEV)
    qd = W.lookup_batch_torch(cfg, keys_d, 0, nl)
    ix.lookup(qd, out)
    torch.cuda.synchronize()
    # sampled cross-check of the generator's queries and of the closed form vs the oracle
    mp = MapOracle(keys, vals)
    idx = np.sort(np.random.default_rng(3).choice(nl, 300_000, replace=False))
    ti = torch.from_numpy(idx).to(DEV)
    qs = W.lookup_at(cfg, keys, idx)
    assert np.array_equal(_u64(qd[ti]), qs)
    assert np.array_equal(_u64(out[ti]), mp.lookup(qs))
    del qd
    vals_d = torch.from_numpy(vals.view(np.int64)).to(DEV)
    hits = 0
    for s0 in range(0, nl, 1 << 27):
        j = torch.arange(s0, s0 + (1 << 27), dtype=torch.int64, device=DEV)
        hit = W._t_ult(W.splitmix64_torch(W.SEED_QUERIES + 3, 2 * j), 1 << 63)
        pick = W._t_umod(W.splitmix64_torch(W.SEED_QUERIES + 3, 2 * j + 1), n)
        exp = torch.where(hit, vals_d[pick], torch.full_like(j, -1))
        assert torch.equal(out[s0: s0 + (1 << 27)], exp), f"lookup mismatch in [{s0}, {s0 + (1 << 27)})"
        hits += int(hit.sum().item())
    assert abs(hits / nl - 0.5) < 0.001
    del out
    # the update batch, then the full post-update state
    uk, uv = W.update_batch_torch(cfg, keys_d)
    ix.update(uk, uv)
    out2 = torch.empty(n, dtype=torch.int64, device=DEV)
    ix.lookup(keys_d, out2)
    torch.cuda.synchronize()
    assert ix.get_error() == 0
    mp.update(_u64(uk), _u64(uv))
    assert mp.last_rejected == 0
    assert np.array_equal(_u64(out2), mp.lookup(keys))
    post = ix.dump()
    for t in (1, 2, 3, 4):
        assert np.array_equal(post["buf"][t], pre["buf"][t]), f"inner buffer {t} changed"
    assert np.array_equal(post["lut"], pre["lut"])
    assert post["root"] == pre["root"]
    leaf = post["buf"][5].reshape(-1, 16)
    assert np.array_equal(leaf[:, :8], pre["buf"][5].reshape(-1, 16)[:, :8])
    assert np.array_equal(np.ascontiguousarray(leaf[:, :8]).view(">u8").ravel().astype(np.uint64), mp.rows)
    assert np.array_equal(np.ascontiguousarray(leaf[:, 8:]).view(np.uint64).ravel(), mp.values)
    pre_v = np.ascontiguousarray(pre["buf"][5].reshape(-1, 16)[:, 8:]).view(np.uint64).ravel()
    assert int((pre_v != mp.values).sum()) > n // 2        # the batch rewrote ~60% of the leaves
    ix.close()


def test_c4_strings_scaled():
    """Config-4 recipe (hierarchical skewed prefixes, 8-32 B keys, Zipf lookups) at
    2^20 keys / 2^22 lookups, element by element vs the pointer-ART oracle."""
    cfg = W.CONFIGS["c4"]
    slots, lens = W.string_keys(4, 1 << 20)
    vals = W.values_for(W.SEED_VALUES + 4, np.arange(1 << 20, dtype=np.uint64))
    o = ArtOracle((slots, lens), vals)
    ix = C.Index((slots, lens), vals)
    st = ix.stats()
    os_ = o.stats()
    assert (st["n4"], st["n16"], st["n48"], st["n256"]) == (os_["n4"], os_["n16"], os_["n48"], os_["n256"])
    assert st["leaf16"] > 0 and st["leaf32"] > 0
    sd, ld = torch.from_numpy(slots).to(DEV), torch.from_numpy(lens).to(DEV)
    qs, ql = W.string_lookup_torch(cfg, sd, ld, 0, 1 << 22)
    out = torch.empty(1 << 22, dtype=torch.int64, device=DEV)
    ix.lookup((qs, ql), out)
    torch.cuda.synchronize()
    qn = (qs.cpu().numpy(), ql.cpu().numpy())
    exp = o.lookup(qn)
    assert np.array_equal(_u64(out), exp)
    assert not np.any(exp == OART_MISS)                      # 100% hit
    # perturbed queries: one flipped byte / truncated length -> misses where absent
    pq = qn[0][:100_000].copy()
    pq[:, 3] ^= 1
    pl = qn[1][:100_000].copy()
    pl[::2] -= 1
    out2 = torch.empty(100_000, dtype=torch.int64, device=DEV)
    ix.lookup((torch.from_numpy(pq).to(DEV), torch.from_numpy(pl).to(DEV)), out2)
    torch.cuda.synchronize()
    assert np.array_equal(_u64(out2), o.lookup((pq, pl)))
    # updates with string keys
    ui = np.random.default_rng(1).integers(0, 1 << 20, 300_000)
    uv = np.random.default_rng(2).integers(0, 2**63, 300_000, dtype=np.uint64)
    ix.update((torch.from_numpy(slots[ui]).to(DEV), torch.from_numpy(lens[ui]).to(DEV)), _t(uv))
    o.update((slots[ui], lens[ui]), uv)
    assert to_records(ix.dump()) == o.dump_structure().tolist()
    ix.close()


@pytest.mark.slow
def test_c4_full_size_every_lookup():
    """Config 4 at full size (2^25 Zipf-prefixed strings, one 2^29-query lookup call
    as the bench times it): EVERY lookup against its closed form from the generator
    (query j is key #idx_j of the set, 100% hit, so its value is vals[idx_j]), and a
    200K sample against the plain-map oracle (pins the closed form to the oracle)."""
    cfg = W.CONFIGS["c4"]
    n = cfg.n_keys
    slots, lens = W.string_keys(4, n)
    vals = W.values_for(W.SEED_VALUES + 4, np.arange(n, dtype=np.uint64))
    ix = C.Index((slots, lens), vals)
    sd, ld = torch.from_numpy(slots).to(DEV), torch.from_numpy(lens).to(DEV)
    nl = cfg.n_lookups
    qidx = W.string_lookup_index_torch(cfg, n, 0, nl, DEV, W.zipf_cdf_torch(n, DEV), W.rank_permutation_torch(cfg, n, DEV))
    qs, ql = sd[qidx], ld[qidx]
    out = torch.empty(nl, dtype=torch.int64, device=DEV)
    ix.lookup((qs, ql), out)
    torch.cuda.synchronize()
    vals_d = torch.from_numpy(vals.view(np.int64)).to(DEV)
    assert torch.equal(out, vals_d[qidx])
    idx = np.sort(np.random.default_rng(4).choice(nl, 200_000, replace=False))
    ti = torch.from_numpy(idx).to(DEV)
    assert np.array_equal(qidx[ti].cpu().numpy(), W.string_lookup_at(cfg, n, idx))
    mp = MapOracle((slots, lens), vals)
    assert np.array_equal(_u64(out[ti]), mp.lookup((qs[ti].cpu().numpy(), ql[ti].cpu().numpy())))
    ix.close()


@pytest.mark.parametrize("kind", ["u64", "u64p", "u32", "bytes"])
def test_prebucket_equals_direct(kind):
    """a5 pre-bucketing only reorders the batch: results identical to the direct
    kernel and to the oracle, for ragged batch sizes across the tile size.  Integer
    kinds also run the bucketed walk with the bucket's root-table slice in shared
    memory (k_lookup_slice), including queries outside every slice (u64p: all keys
    share the top byte 0x7F, half the queries do not; u32: 10% of the queries
    leave the keys' common prefix byte 0x00)."""
    lut = 0 if kind == "bytes" else 3
    if kind == "u64":
        cfg = W.CONFIGS["c1"]
        keys, vals = W.build_set(cfg)
        mk = lambda m: W.lookup_batch(cfg, keys, 0, m)
    elif kind == "u64p":
        rng = np.random.default_rng(3)
        keys = np.unique(rng.integers(0, 1 << 56, 1 << 17, dtype=np.uint64) | np.uint64(0x7F << 56))
        vals = np.arange(keys.shape[0], dtype=np.uint64) * 3 + 1

        def mk(m):
            hit = keys[rng.integers(0, keys.shape[0], m)]
            other = rng.integers(0, 2**63, m, dtype=np.uint64) * np.uint64(2) + np.uint64(1)
            return np.where(rng.random(m) < 0.5, hit, other)
    elif kind == "u32":
        keys = (np.arange(1 << 18, dtype=np.uint32) * 13) & np.uint32(0xFFFFFF)
        keys = np.unique(keys)
        vals = np.arange(keys.shape[0], dtype=np.uint64) + 1
        rng = np.random.default_rng(0)
        mk = lambda m: np.where(rng.random(m) < 0.9, rng.integers(0, 1 << 24, m, dtype=np.uint32),
                                rng.integers(0, 1 << 32, m, dtype=np.uint32)).astype(np.uint32)
    else:
        keys = W.string_keys(4, 1 << 16)
        vals = np.arange(1 << 16, dtype=np.uint64) + 5
        mk = lambda m: (lambda idx: (keys[0][idx].copy(), keys[1][idx].copy()))(
            W.string_lookup_at(W.CONFIGS["c4"], 1 << 16, np.arange(m)))
    mp = MapOracle(keys, vals)
    off = C.Index(keys, vals, lut_bytes=lut, prebucket=C.PREBUCKET_OFF)
    variants = [C.Index(keys, vals, lut_bytes=lut, prebucket=C.PREBUCKET_ON, slice_lut=C.SLICE_OFF)]
    if kind != "bytes":
        variants.append(C.Index(keys, vals, lut_bytes=lut, prebucket=C.PREBUCKET_ON, slice_lut=C.SLICE_ON))
        variants.append(C.Index(keys, vals, lut_bytes=lut, prebucket=C.PREBUCKET_ON, wide_lut=C.WIDE_ON))
        variants.append(C.Index(keys, vals, lut_bytes=lut, prebucket=C.PREBUCKET_ON, wide_lut=C.WIDE_OFF))
        # the global K-BUCKET form (hist + scatter) beside the default tile form
        for wl in (C.WIDE_ON, C.WIDE_OFF):
            variants.append(C.Index(keys, vals, lut_bytes=lut, prebucket=C.PREBUCKET_ON, wide_lut=wl,
                                    bucket_form=C.BUCKET_GLOBAL))
    # 2048 * 4096 + 4097 spans more than one pass of k_bscan_rows (2048 tiles per pass)
    sizes = (4095, 4096, 4097, 100_003, 1 << 20) + ((2048 * 4096 + 4097,) if kind == "u64" else ())
    for m in sizes:
        q = mk(m)
        b = _lookup(off, q)
        assert np.array_equal(b, mp.lookup(q)), m
        for on in variants:
            assert np.array_equal(_lookup(on, q), b), m
    for ix in [off] + variants:
        ix.close()


@pytest.mark.parametrize("kind", ["u64", "u32", "bytes"])
def test_prebucket_updates_equal_direct(kind):
    """Pre-bucketed update batches keep the ORIGINAL op index as priority:
    same final state as the direct kernels and the sequential oracle, with many
    duplicate keys spread over different tiles and buckets."""
    rng = np.random.default_rng(9)
    if kind == "u64":
        keys, vals = W.build_set(W.CONFIGS["c1"])
    elif kind == "u32":
        keys = np.unique((np.arange(1 << 17, dtype=np.uint32) * 29) & np.uint32(0xFFFFFF))
        vals = np.arange(keys.shape[0], dtype=np.uint64) + 1
    else:
        keys = W.string_keys(4, 1 << 15)
        vals = np.arange(1 << 15, dtype=np.uint64) + 5
    n = keys[1].shape[0] if isinstance(keys, tuple) else keys.shape[0]
    on = C.Index(keys, vals, prebucket=C.PREBUCKET_ON)
    off = C.Index(keys, vals, prebucket=C.PREBUCKET_OFF)
    mp = MapOracle(keys, vals)
    wide = C.Index(keys, vals, prebucket=C.PREBUCKET_ON, lut_bytes=0 if kind == "bytes" else 3, wide_lut=C.WIDE_ON)
    for m in (4097, 200_003):
        pick = rng.integers(0, min(n, 3000), m)                     # heavy duplication
        uk = (keys[0][pick].copy(), keys[1][pick].copy()) if isinstance(keys, tuple) else keys[pick].copy()
        uv = rng.integers(0, 2**63, m, dtype=np.uint64)
        on.update(_t(uk), _t(uv))
        off.update(_t(uk), _t(uv))
        wide.update(_t(uk), _t(uv))
        mp.update(uk, uv)
        a, b = _lookup(on, keys), _lookup(off, keys)
        assert np.array_equal(a, b) and np.array_equal(a, mp.lookup(keys)), m
        assert np.array_equal(_lookup(wide, keys), a), m
    on.close()
    off.close()
    wide.close()


@pytest.mark.parametrize("on_stream", [False, True])
def test_l2_persist_window_results_identical(on_stream):
    """cuart_build_opts.l2_persist (keep the merged upper layers cached) sets a
    persisting access-policy window over the root tables for the launches of each
    call; it changes performance only: results equal the oracle, on the legacy and on
    a created stream (whose previous policy is restored)."""
    cfg = W.CONFIGS["c1"]
    keys, vals = W.build_set(cfg)
    ix = C.Index(keys, vals, lut_bytes=3, l2_persist=1, prebucket=C.PREBUCKET_ON)
    assert ix.stats()["l2_window_bytes"] > 0
    o = MapOracle(keys, vals)
    q = W.lookup_batch(cfg, keys)
    s = torch.cuda.Stream() if on_stream else torch.cuda.current_stream()
    with torch.cuda.stream(s):
        got = _lookup(ix, q)
        uk, uv = W.update_batch(cfg, keys)
        ix.update(_t(uk), _t(uv))
        got2 = _lookup(ix, keys)
    assert np.array_equal(got, o.lookup(q))
    o.update(uk, uv)
    assert np.array_equal(got2, o.lookup(keys))
    ix.close()


@pytest.mark.parametrize("prebucket", [1, 2])
def test_epoch_wrap(prebucket):
    """§8(a) a9: the conflict words carry the batch epoch in their high half, so no
    reset pass runs between batches; every 2^32 - 2 batches the epoch wraps, the words
    are cleared and the epoch restarts at 1.  Driven through the test hook: batches
    before, across and after the wrap (duplicate-heavy, so stale high-priority words
    of the last pre-wrap batch would block later winners if the clear were missing)
    equal the sequential oracle."""
    cfg = W.CONFIGS["c1"]
    keys, vals = W.build_set(cfg)
    ix = C.Index(keys, vals, lut_bytes=3, prebucket=prebucket)
    o = MapOracle(keys, vals)
    B = C._binding
    B._check(B.lib().cuart_debug_set_epoch(ix.h, 0xFFFFFFFC), "cuart_debug_set_epoch")
    rng = np.random.default_rng(17)
    for b in range(5):
        m = 60_000 if b % 2 == 0 else 5_000         # a small batch after a big one: low op indices
        uk = keys[rng.integers(0, 2000, m)]           # few distinct keys, many duplicates
        uv = rng.integers(0, 2**63, m, dtype=np.uint64)
        ix.update(_t(uk), _t(uv))
        o.update(uk, uv)
        assert np.array_equal(_lookup(ix, keys), o.lookup(keys)), b
    ix.close()


def test_host_pipeline_orders_after_async_update():
    """the host-buffer calls run on the index's non-blocking streams; an
    asynchronous cuart_update enqueued just before on the legacy stream must be
    visible to them (they join the legacy stream at entry)."""
    cfg = W.CONFIGS["c1"]
    keys, vals = W.build_set(cfg)
    ix = C.Index(keys, vals, lut_bytes=3)
    o = MapOracle(keys, vals)
    for rep in range(3):
        uk, uv = W.update_batch(cfg, keys, rep * 100_000, 100_000)
        ix.update(_t(uk), _t(uv), stream=0)           # async, legacy stream, no synchronisation
        o.update(uk, uv)
        assert np.array_equal(ix.lookup_host(keys), o.lookup(keys)), rep
        uk2, uv2 = W.update_batch(cfg, keys, 10**6 + rep * 50_000, 50_000)
        ix.update_host(uk2, uv2)
        o.update(uk2, uv2)
    out = torch.empty(keys.shape[0], dtype=torch.int64, device=DEV)
    ix.lookup(_t(keys), out, stream=0)
    torch.cuda.synchronize()
    assert np.array_equal(_u64(out), o.lookup(keys))
    ix.close()
