"""C-ABI library checks that need no GPU: exports, error mapping, host builder
and the CPU layout walker against the oracle."""
import random
import re
import os

import numpy as np
import pytest

import paper_conf_icpp_koppehelggp21_b200 as C
from oracle import ArtOracle, MapOracle, OART_MISS
from tests.artspec import golden_key, load_golden
from tests.layout_decode import REC, split_link, to_records

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
MISS = int(OART_MISS)


def test_library_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "cuart.h")).read()
    names = sorted(set(re.findall(r"\b(cuart_[a-z_0-9]+)\s*\(", hdr)))
    assert "cuart_build" in names and "cuart_lookup" in names and "cuart_update" in names and "cuart_destroy" in names
    lib = C.lib()
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing, missing
    assert C.cuart_status_string(0) == "ok"
    assert C.cuart_status_string(3) == "key set is not prefix-free"


def test_record_sizes_match_paper_node_sizes():
    # "650B for N48 and 2KB for N256" -> 16-B header + index + 8-B links
    assert abs(REC[3] - 650) < 32 and REC[3] % 32 == 0
    assert abs(REC[4] - 2048) < 40 and REC[4] % 32 == 0
    # P:108/P:110 alignment: every record a multiple of 16, large ones of 32
    assert all(v % 16 == 0 for v in REC.values())


def test_errors_without_gpu():
    with pytest.raises(C.CuartError) as e:
        C.cuart_layout_build(np.array([1, 2], np.uint64), np.array([1, C.CUART_MISS], np.uint64))
    assert e.value.status == 4
    s = np.zeros((2, 32), np.uint8)
    s[0, :2] = [97, 98]
    s[1, :3] = [97, 98, 99]
    with pytest.raises(C.CuartError) as e:
        C.cuart_layout_build((s, np.array([2, 3], np.uint8)), np.array([1, 2], np.uint64))
    assert e.value.status == 3
    with pytest.raises(C.CuartError) as e:
        C.cuart_layout_build((s, np.array([2, 33], np.uint8)), np.array([1, 2], np.uint64))
    assert e.value.status == 2
    with pytest.raises(C.CuartError) as e:
        C.cuart_layout_build((s, np.array([0, 3], np.uint8)), np.array([1, 2], np.uint64))
    assert e.value.status == 2
    with pytest.raises(C.CuartError) as e:
        C.cuart_layout_build(np.array([1], np.uint64), np.array([1], np.uint64), lut_bytes=4)
    assert e.value.status == 1


def test_cuart_build_without_device_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(C.CuartError) as e:
        C.cuart_build(np.array([1, 2], np.uint64), np.array([1, 2], np.uint64))
    assert e.value.status == 8


def test_dist_cfg_validation_without_gpu():
    """cuart_dist_build / cuart_dist_partition / cuart_dist_chunk_plan reject bad
    configurations before touching a device; a valid one reaches the device check."""
    import ctypes
    import torch
    from paper_conf_icpp_koppehelggp21_b200 import dist as D
    keys = np.arange(1000, dtype=np.uint64) * np.uint64(7919)
    vals = np.arange(1000, dtype=np.uint64)
    k, n, keep = C._binding.make_keys(keys)

    def build(**kw):
        c, keep2 = D._cfg(kw.get("rank", 0), kw.get("world", 2), "range", "p2p", None,
                          splitters=kw.get("splitters"), keys_local=kw.get("keys_local", False))
        for f in ("nranks", "mode", "transport"):
            if f in kw:
                setattr(c, f, kw[f])
        h = ctypes.c_void_p()
        return D.lib().cuart_dist_build(ctypes.byref(c), ctypes.byref(k), vals.ctypes.data, n, ctypes.byref(h))

    assert build(rank=2) == 1                                   # rank out of range
    assert build(nranks=17) == 1                                # more ranks than CUART_DIST_MAX_RANKS
    assert build(mode=7) == 1 and build(transport=9) == 1
    assert build(world=3, splitters=np.array([5, 3], np.uint64)) == 1        # descending splitters
    assert build(keys_local=True) == 1                          # a local share needs its splitters
    if not torch.cuda.is_available():
        assert build(world=1) == 8                              # valid: CUART_ERR_NO_DEVICE here
    M = np.ones((2, 2), np.uint64)
    bad = np.zeros(3, np.uint64)
    assert D.lib().cuart_dist_chunk_plan(2, 2, M.ctypes.data, bad.ctypes.data, bad.ctypes.data, bad.ctypes.data) == 1
    assert D.lib().cuart_dist_chunk_plan(0, 0, M.ctypes.data, bad.ctypes.data, bad.ctypes.data, bad.ctypes.data) == 1
    sp, own = D.partition(keys, 0, 4)
    assert np.all(np.diff(sp.astype(np.float64)) >= 0) and set(own.tolist()) == {0, 1, 2, 3}


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


@pytest.mark.parametrize("name", ["ex_a_u64.json", "ex_d_strings.json", "ex_e_prefix_split.json", "ex_f_long_prefix.json"])
def test_golden_layout(name):
    g = load_golden(name)
    kind = g["kind"]
    keys = [golden_key(kind, k) for k in g["keys"]]
    inp = _as_input(kind, keys)
    vals = np.array(g["values"], np.uint64)
    o = ArtOracle(inp, vals)
    for lut in (0, 1, 2, 3):
        lay = C.Layout(inp, vals, lut_bytes=lut)
        assert to_records(lay.view()) == o.dump_structure().tolist()
        qs = [golden_key(kind, q) for q, _ in g["lookups"]]
        exp = [MISS if v is None else v for _, v in g["lookups"]]
        if kind == "bytes":
            got = lay.lookup(_strings(qs)).tolist()
        else:
            got = lay.lookup(_as_input(kind, qs)).tolist()
        assert got == exp


def _random_set(rng, n, mode):
    s = set()
    while len(s) < n:
        if mode == "u64":
            s.add(rng.getrandbits(64).to_bytes(8, "big"))
        elif mode == "u64_shared":
            k = bytearray(8)
            lead = rng.randrange(0, 8)
            for i in range(lead, 8):
                k[i] = rng.choice([0, 0xFF, rng.randrange(256), rng.randrange(3)])
            s.add(bytes(k))
        elif mode == "u32":
            s.add(rng.choice([rng.getrandbits(32), rng.getrandbits(12)]).to_bytes(4, "big"))
        else:
            stem = rng.choice([b"", b"a", b"ab", b"q" * 14, b"r" * 15, b"s" * 16, b"t" * 24])
            body = bytes(rng.choice(b"abz\x01\xff") for _ in range(rng.randrange(0, 31 - len(stem) + 1)))
            s.add((stem + body)[:31] + b"\x00")
    return sorted(s)


@pytest.mark.parametrize("mode", ["u64", "u64_shared", "u32", "bytes"])
@pytest.mark.parametrize("seed", range(5))
def test_builder_matches_oracle_structure_and_lookups(mode, seed):
    rng = random.Random(seed * 31 + len(mode))
    n = rng.choice([0, 1, 2, 4, 5, 16, 17, 48, 49, 256, 300, 3000])
    keys = _random_set(rng, n, mode)
    rng.shuffle(keys)
    vals = np.array([rng.getrandbits(63) for _ in keys], np.uint64)
    kind = "bytes" if mode == "bytes" else ("u32" if mode == "u32" else "u64")
    inp = _as_input(kind, keys) if keys else (np.zeros(0, np.uint64) if kind == "u64" else np.zeros(0, np.uint32) if kind == "u32" else (np.zeros((0, 32), np.uint8), np.zeros(0, np.uint8)))
    o = ArtOracle(inp, vals)
    probes = list(keys)
    for k in keys[:100]:
        flip = bytearray(k)
        flip[rng.randrange(len(k))] ^= 1 << rng.randrange(8)
        probes.append(bytes(flip))
        if kind == "bytes":
            probes += [k[:-1] or b"\x01", k[:-1] + b"\x02"]
    probes += [rng.getrandbits(64 if kind != "u32" else 32).to_bytes(8 if kind != "u32" else 4, "big") for _ in range(64)]
    if kind != "bytes":
        probes = [p for p in probes if len(p) == (8 if kind == "u64" else 4)]
    pin = _as_input(kind, probes)
    exp = o.lookup(pin) if probes else np.zeros(0, np.uint64)
    for lut in (0, 1, 2, 3):
        lay = C.Layout(inp, vals, lut_bytes=lut)
        view = lay.view()
        assert to_records(view) == o.dump_structure().tolist()
        if probes:
            assert np.array_equal(lay.lookup(pin), exp)
        if lut:
            assert view["lut"].shape[0] == 1 << (8 * lut)
    # leaves: lexicographic rank within their size class
    cls = {}
    for k in sorted(keys):
        t = 5 if len(k) <= 8 else 6 if len(k) <= 16 else 7
        cls.setdefault(t, []).append(k)
    view = C.Layout(inp, vals).view()
    for t, ks in cls.items():
        assert view["count"][t] == len(ks)
        recs = view["buf"][t].reshape(-1, view["record_bytes"][t])
        for i, k in enumerate(ks):
            assert bytes(recs[i, : len(k)]) == k


def test_lut_size_and_entries_c1():
    import workloads as W
    cfg = W.CONFIGS["c1"]
    keys, vals = W.build_set(cfg)
    lay = C.Layout(keys, vals, lut_bytes=3)
    v = lay.view()
    assert v["lut"].nbytes == 128 * 1024 * 1024       # 2^24 links = 128 MB
    nz = v["lut"][v["lut"] != 0]
    # c1: 65,536 random keys -> every used 3-byte prefix points at a leaf or an N4/N16 below depth 3
    types = np.unique(nz >> np.uint64(60))
    assert set(types.tolist()) <= {1, 2, 5}
    q = W.lookup_batch(cfg, keys, 0, 100_000)
    mp = MapOracle(keys, vals)
    assert np.array_equal(lay.lookup(q), mp.lookup(q))
    assert np.array_equal(C.Layout(keys, vals, 0).lookup(q), mp.lookup(q))


def test_c1_stats_shape():
    import workloads as W
    keys, vals = W.build_set(W.CONFIGS["c1"])
    v = C.Layout(keys, vals).view()
    o = ArtOracle(keys, vals).stats()
    assert v["count"][1:5] == [o["n4"], o["n16"], o["n48"], o["n256"]]
    assert v["count"][5] == 65_536
    assert split_link(v["root"])[0] == 4   # root N256


def test_duplicates_last_wins_in_build():
    lay = C.Layout(np.array([5, 6, 5, 7, 5], np.uint64), np.array([1, 2, 3, 4, 9], np.uint64))
    assert lay.lookup(np.array([5, 6, 7, 8], np.uint64)).tolist() == [9, 2, 4, MISS]


def test_query_bytes_past_length_are_ignored():
    slots, lens = _strings([b"ab\x00", b"abc\x00"])
    lay = C.Layout((slots, lens), np.array([1, 2], np.uint64))
    q = np.full((3, 32), 0xEE, np.uint8)
    q[0, :3] = [97, 98, 0]
    q[1, :4] = [97, 98, 99, 0]
    q[2, :2] = [97, 98]
    assert lay.lookup((q, np.array([3, 4, 2], np.uint8))).tolist() == [1, 2, MISS]


def test_dense_u32_shape():
    n = 1 << 18
    keys = np.arange(n, dtype=np.uint32)
    v = C.Layout(keys, keys.astype(np.uint64) + 1, lut_bytes=3).view()
    # root N4? no: keys 0..2^18-1 -> byte0=0 shared, byte1 in 0..3 -> root N4 prefix [00] depth 1
    t, aux, _ = split_link(v["root"])
    assert (t, aux) == (1, 1)
    assert v["count"][4] == 4 + 1024 and v["count"][5] == n
    q = np.array([0, 5, n - 1, n, 1 << 30], np.uint32)
    assert C.Layout(keys, keys.astype(np.uint64) + 1, lut_bytes=3).lookup(q).tolist() == [1, 6, n, MISS, MISS]


def test_sector_walker_wide_root_table():
    """cuart_layout_sectors_ex(WIDE) counts the path of the pre-bucketed walk that
    starts from the wide root table: the 32-B entry carries the target N16's keys,
    so the N16 key sector disappears, and when all of the N16's children are leaves
    (consecutive in the ordered leaf buffer) the entry's leaf run replaces the
    child-link read too (hand count: LUT + N16 keys + child + leaf = 4 sectors plain,
    LUT + leaf = 2 wide; a missing last byte 2 vs 1).  With one inner child the run
    is absent and the wide walk reads the child link: LUT + child + leaf = 3."""
    keys = (np.uint32(0x01020300) + np.arange(10, dtype=np.uint32)).astype(np.uint32)
    lay = C.Layout(keys, np.arange(10, dtype=np.uint64) + 1, lut_bytes=3)
    q = np.array([0x01020305, 0x010203F0], np.uint32)
    assert lay.sectors(q).tolist() == [4, 2]
    assert lay.sectors(q, wide=True).tolist() == [2, 1]
    lay.close()
    base = np.uint64(0x0102030000000000)
    keys = np.concatenate([base + (np.arange(10, dtype=np.uint64) << np.uint64(32)),
                           base + np.array([0x0A00000001, 0x0A00000002], np.uint64)])
    lay = C.Layout(keys, np.arange(12, dtype=np.uint64) + 1, lut_bytes=3)
    q = np.array([base + np.uint64(5 << 32), base + np.uint64(0xF0 << 32)], np.uint64)
    assert lay.lookup(q).tolist() == [6, MISS]
    assert lay.sectors(q).tolist() == [4, 2]
    assert lay.sectors(q, wide=True).tolist() == [3, 1]
    lay.close()
    # dense u32 (c2 shape): LUT[3 bytes] -> a full N256 whose 256 children are leaves,
    # so the wide entry's run gives the leaf directly: LUT + N256 child + leaf = 3
    # plain, LUT + leaf = 2 wide; an absent 3-byte prefix misses at the LUT (1).
    keys = np.arange(1 << 16, dtype=np.uint32)
    lay = C.Layout(keys, keys.astype(np.uint64) + 1, lut_bytes=3)
    q = np.array([5, 70000, 65535], np.uint32)
    assert lay.lookup(q).tolist() == [6, MISS, 65536]
    assert lay.sectors(q).tolist() == [3, 1, 3]
    assert lay.sectors(q, wide=True).tolist() == [2, 1, 2]
    lay.close()


def test_sector_walker_skip_table_path():
    """cuart_layout_sectors_ex(SKIP(D)) counts the byte-string walk that starts from
    the skip table: one 32-B probe, then only the levels below the node covering the
    query's first D bytes.  Hand case: keys "aaaaaaa" + x + "b" (x in 0..4, length 9)
    and "zz" (length 2): the root N4 branches at byte 0; under "a" an N16 (5 children)
    branches at depth 7 over leaf16 records.  Plain walk = root N4 (1 sector) + N16 keys
    and child (2) + leaf16 (1) = 4; skip D = 8: probe (1) + leaf (1) = 2; D = 4: probe +
    N16 (2) + leaf = 4 (the N16 branches at depth 7 >= 4, so it covers "aaaa"); a query
    shorter than D takes the plain walk (zz: root N4 + leaf8 = 2); "aaaabbbbb" has the
    prefix but misses at the N16's keys (probe + 1 = 2); "qqqqq" has no 4-byte prefix in
    the tree and stops at the probe (1)."""
    names = [b"aaaaaaa" + bytes([0x30 + x]) + b"b" for x in range(5)] + [b"zz"]
    slots = np.zeros((len(names), 32), np.uint8)
    for i, s in enumerate(names):
        slots[i, :len(s)] = np.frombuffer(s, np.uint8)
    lens = np.array([len(s) for s in names], np.uint8)
    lay = C.Layout((slots, lens), np.arange(len(names), dtype=np.uint64) + 1, lut_bytes=0)
    q_names = [names[2], b"zz", b"aaaabbbbb", b"qqqqq"]
    qs = np.zeros((4, 32), np.uint8)
    for i, s in enumerate(q_names):
        qs[i, :len(s)] = np.frombuffer(s, np.uint8)
    ql = np.array([len(s) for s in q_names], np.uint8)
    assert lay.lookup((qs, ql)).tolist()[:2] == [3, 6]
    plain = lay.sectors((qs, ql)).tolist()
    assert plain[:2] == [4, 2]
    assert lay.sectors((qs, ql), skip_prefix=8).tolist()[:2] == [2, 2]
    assert lay.sectors((qs, ql), skip_prefix=4).tolist() == [4, 2, 2, 1]
    lay.close()
