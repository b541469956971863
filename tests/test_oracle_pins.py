"""Pins for the CPU oracle (runs without a GPU).

The oracle (oracle/art_oracle.c, oracle/art.py) is checked against things other
than itself: hand-derived golden trees (tests/golden/, each with its citation),
closed-form special cases, brute force (Python dict / sorted list) on tiny
inputs, an independent recursive-partition construction of the canonical ART,
ART invariants, and insertion-order independence.  Each is chosen so that a
plausible mistake (a dropped prefix byte, a wrong depth, wrong growth threshold,
unsorted children, a lost update ordering) fails at least one of them.
"""
import random

import numpy as np
import pytest

from oracle import ArtOracle, MapOracle, OART_MISS
from tests.artspec import (canonical_records, check_invariants, golden_key, golden_tree_records,
                           load_golden, node_type_for)

MISS = int(OART_MISS)
GOLDENS = ["ex_a_u64.json", "ex_d_strings.json", "ex_e_prefix_split.json", "ex_f_long_prefix.json"]


def _as_input(kind, keys):
    if kind == "u64":
        return np.array([int.from_bytes(k, "big") for k in keys], dtype=np.uint64)
    if kind == "u32":
        return np.array([int.from_bytes(k, "big") for k in keys], dtype=np.uint32)
    slots = np.zeros((len(keys), 32), dtype=np.uint8)
    lens = np.zeros(len(keys), dtype=np.uint8)
    for i, k in enumerate(keys):
        slots[i, : len(k)] = np.frombuffer(k, dtype=np.uint8)
        lens[i] = len(k)
    return slots, lens


# ------------------------------------------------------------------ golden trees
@pytest.mark.parametrize("name", GOLDENS)
def test_golden_structure_lookup_update(name):
    g = load_golden(name)
    kind = g["kind"]
    keys = [golden_key(kind, k) for k in g["keys"]]
    o = ArtOracle(_as_input(kind, keys), np.array(g["values"], dtype=np.uint64))
    assert o.dump_structure().tolist() == golden_tree_records(g["tree"])
    st = o.stats()
    for k, v in g["stats"].items():
        assert st[k] == v
    qs = [golden_key(kind, q) for q, _ in g["lookups"]]
    exp = [MISS if v is None else v for _, v in g["lookups"]]
    if kind == "bytes":
        got = [o.lookup_one(q) for q in qs]   # includes queries of other lengths
    else:
        got = o.lookup(_as_input(kind, qs)).tolist()
    assert got == exp
    uk = [golden_key(kind, k) for k, _ in g["update_ops"]]
    uv = np.array([v for _, v in g["update_ops"]], dtype=np.uint64)
    o.update(_as_input(kind, uk), uv)
    for k, v in g["after_update"]:
        assert o.lookup_one(golden_key(kind, k)) == v


# ------------------------------------------------------------------ closed forms
@pytest.mark.parametrize("m,exp_type", [(1, 0), (2, 1), (4, 1), (5, 2), (16, 2), (17, 3), (48, 3), (49, 4), (256, 4)])
def test_ex_b_thresholds(m, exp_type):
    """Ex-B: keys {i * 2^56 : i < m} -> root type by child count; all children leaves."""
    keys = np.array([i << 56 for i in range(m)], dtype=np.uint64)
    o = ArtOracle(keys, np.arange(m, dtype=np.uint64) + 1)
    rec = o.dump_structure().tolist()
    assert rec[0] == exp_type
    st = o.stats()
    assert st["leaves"] == m
    if m == 1:
        assert st["height"] == 1
    else:
        assert st["height"] == 2
        assert sum(st[t] for t in ("n4", "n16", "n48", "n256")) == 1
        assert rec[1] == 0 and rec[2] == m and rec[3: 3 + m] == list(range(m))


def test_ex_c_dense_u32_small():
    """Ex-C (scaled to 2^16): keys 0..2^16-1 as u32 -> root N256 with prefix [00 00]
    branching at depth 2, 256 N256 children (prefix empty), 2^16 leaves."""
    n = 1 << 16
    o = ArtOracle(np.arange(n, dtype=np.uint32), np.arange(n, dtype=np.uint64) * 3 + 1)
    st = o.stats()
    assert st == {"leaves": n, "n4": 0, "n16": 0, "n48": 0, "n256": 257, "height": 3}
    rec = o.dump_structure()
    assert rec[:4].tolist() == [4, 2, 0, 0] and rec[4] == 256
    q = np.array([0, 1, 255, 256, 65535, 65536, 1 << 24, 0xFFFFFFFF], dtype=np.uint32)
    assert o.lookup(q).tolist() == [1, 4, 766, 769, 65535 * 3 + 1, MISS, MISS, MISS]


def test_ex_c_full_stats_closed_form_with_map():
    """Ex-C via the plain map at the full 2^24 size: dense keys give lookup(k)=v(k) for all k."""
    n = 1 << 24
    keys = np.arange(n, dtype=np.uint32)
    vals = keys.astype(np.uint64) * 7 + 5
    m = MapOracle(keys, vals)
    q = np.array([0, 1, n - 1, n, n + 1, 0xFFFFFFFF], dtype=np.uint32)
    assert m.lookup(q).tolist() == [5, 12, (n - 1) * 7 + 5, MISS, MISS, MISS]


# ------------------------------------------------------------------ random sets vs brute force
def _random_keyset(rng, n, mode):
    s = set()
    while len(s) < n:
        if mode == "u64":
            s.add(rng.getrandbits(64).to_bytes(8, "big"))
        elif mode == "u64_shared":       # keys sharing 0..7 leading bytes, 0x00/0xFF heavy
            base = bytearray(rng.choice([b"\x00" * 8, b"\xff" * 8, bytes(8)]))
            k = rng.randrange(0, 8)
            for i in range(k, 8):
                base[i] = rng.choice([0, 0xFF, rng.randrange(256), rng.randrange(4)])
            s.add(bytes(base))
        elif mode == "bytes":            # prefix-free via a 0x00 terminator, shared stems
            stem = rng.choice([b"", b"a", b"ab", b"abc", b"x" * 14, b"y" * 15, b"z" * 20])
            body = bytes(rng.choice(b"abcdz\x01\xff") for _ in range(rng.randrange(0, 31 - len(stem) + 1)))
            k = (stem + body)[:31] + b"\x00"
            s.add(k)
    return sorted(s)


@pytest.mark.parametrize("mode", ["u64", "u64_shared", "bytes"])
@pytest.mark.parametrize("seed", range(6))
def test_random_vs_bruteforce_and_canonical(mode, seed):
    rng = random.Random(1000 * seed + hash(mode) % 997)
    n = rng.choice([1, 2, 3, 4, 5, 16, 17, 48, 49, 200, 700])
    keys = _random_keyset(rng, n, mode)
    rng.shuffle(keys)
    vals = [rng.getrandbits(63) for _ in keys]
    ref = dict(zip(keys, vals))
    o = ArtOracle()
    for k, v in zip(keys, vals):
        assert o.insert_one(k, v) == 0
    assert len(o) == len(ref)
    rec = o.dump_structure().tolist()
    # independent construction of the canonical tree
    assert rec == canonical_records(list(ref.items()))
    check_invariants(rec, ref)
    # brute-force lookups: present keys, absent keys, prefixes and extensions of present keys
    probes = list(keys)
    for k in keys[:50]:
        probes += [k[:-1], k + b"\x00", bytes([k[0] ^ 1]) + k[1:], k[:-1] + bytes([k[-1] ^ 0x80])]
    probes += [rng.getrandbits(64).to_bytes(8, "big") for _ in range(50)]
    for q in probes:
        if 1 <= len(q) <= 32:
            assert o.lookup_one(q) == ref.get(q, MISS)
    # in-order dump is the sorted dict
    ks, ls, vs = o.dump_inorder()
    got = [(bytes(ks[i, : ls[i]]), int(vs[i])) for i in range(len(ls))]
    assert got == sorted(ref.items())


@pytest.mark.parametrize("seed", range(4))
def test_insertion_order_independence(seed):
    rng = random.Random(seed)
    keys = _random_keyset(rng, 300, "u64_shared" if seed % 2 else "bytes")
    vals = {k: rng.getrandbits(60) for k in keys}
    dumps = []
    for order in ("sorted", "reversed", "s1", "s2", "s3"):
        ks = list(keys)
        if order == "reversed":
            ks.reverse()
        elif order.startswith("s"):
            random.Random(order).shuffle(ks)
        o = ArtOracle()
        for k in ks:
            o.insert_one(k, vals[k])
        dumps.append(o.dump_structure().tolist())
    assert all(d == dumps[0] for d in dumps)


def test_node_growth_each_threshold():
    """Children added one by one under a fixed prefix: the node type follows 4/16/48."""
    o = ArtOracle()
    for i in range(256):
        o.insert_one(bytes([7, i]), i + 1)
        rec = o.dump_structure().tolist()
        if i == 0:
            assert rec[0] == 0
        else:
            assert rec[0] == node_type_for(i + 1)
            assert rec[1] == 1 and rec[2] == 7   # prefix [07]


# ------------------------------------------------------------------ updates
def test_update_hand_pins():
    k = np.array([1 << 40, 2 << 40, 3 << 40], dtype=np.uint64)
    o = ArtOracle(k, np.array([100, 200, 300], dtype=np.uint64))
    m = MapOracle(k, np.array([100, 200, 300], dtype=np.uint64))
    # batch [(k,1),(k,2),(k,3)] -> 3
    for x in (o, m):
        x.update(np.array([k[0]] * 3, dtype=np.uint64), np.array([1, 2, 3], dtype=np.uint64))
    # op indices 0, 5, 3 on one key -> the index-5 value (highest index wins)
    ops_k = np.array([k[1], k[2], k[2], k[0] + np.uint64(1), k[2], k[1], k[2]], dtype=np.uint64)
    ops_v = np.array([10, 11, 12, 13, 14, 15, 16], dtype=np.uint64)
    for x in (o, m):
        x.update(ops_k, ops_v)
    exp = [3, 15, 16, MISS]
    q = np.array([k[0], k[1], k[2], k[0] + np.uint64(1)], dtype=np.uint64)
    assert o.lookup(q).tolist() == exp
    assert m.lookup(q).tolist() == exp


@pytest.mark.parametrize("seed", range(5))
def test_update_vs_sequential_dict(seed):
    rng = random.Random(77 + seed)
    keys = _random_keyset(rng, 500, ["u64", "bytes", "u64_shared"][seed % 3])
    vals = [rng.getrandbits(62) for _ in keys]
    ref = dict(zip(keys, vals))
    o = ArtOracle()
    for k, v in zip(keys, vals):
        o.insert_one(k, v)
    ops = []
    for _ in range(2000):
        if rng.random() < 0.02:            # reserved value: the op is dropped (reading C5)
            ops.append((rng.choice(keys), MISS))
        elif rng.random() < 0.8:
            ops.append((rng.choice(keys), rng.getrandbits(62)))
        else:
            ops.append((rng.getrandbits(64).to_bytes(8, "big") if rng.random() < 0.5 else b"nope\x00", rng.getrandbits(62)))
    for k, v in ops:                   # brute force: apply in order, present keys only
        if k in ref and v != MISS:
            ref[k] = v
    if all(len(k) == 8 for k, _ in ops) and all(len(k) == 8 for k in keys):
        o.update(np.array([int.from_bytes(k, "big") for k, _ in ops], dtype=np.uint64),
                 np.array([v for _, v in ops], dtype=np.uint64))
    else:
        slots = np.zeros((len(ops), 32), np.uint8)
        lens = np.zeros(len(ops), np.uint8)
        for i, (k, _) in enumerate(ops):
            slots[i, : len(k)] = np.frombuffer(k, np.uint8)
            lens[i] = len(k)
        o.update((slots, lens), np.array([v for _, v in ops], dtype=np.uint64))
    for k in keys:
        assert o.lookup_one(k) == ref[k]


def test_reserved_value_ops_are_dropped():
    """Reading C5 (CUART_MISS is the lookup's absent answer, so it cannot be
    stored): an op carrying it is a no-op -- it neither writes nor wins over an
    earlier op on the same key -- and the rest of the batch applies."""
    k = np.array([1, 2, 3], np.uint64)
    for mk in (ArtOracle, MapOracle):
        x = mk(k, np.array([10, 20, 30], np.uint64))
        x.update(np.array([1, 2], np.uint64), np.array([MISS, 5], np.uint64))
        assert x.lookup(k).tolist() == [10, 5, 30] and x.last_rejected == 1
        x.update(np.array([3, 3, 2], np.uint64), np.array([7, MISS, MISS], np.uint64))
        assert x.lookup(k).tolist() == [10, 5, 7] and x.last_rejected == 2
        # mixed batch (reading C17): a dropped op does not locate, so an earlier op wins;
        # a delete carries no value, so the reserved value does not drop it
        x.apply(np.array([1, 1, 2, 3], np.uint64), np.array([11, MISS, MISS, MISS], np.uint64),
                np.array([0, 0, 1, 0], np.uint8))
        assert x.lookup(k).tolist() == [11, MISS, 7] and x.last_rejected == 2


def test_lookup_mt_equals_single_thread():
    import workloads as W
    cfg = W.CONFIGS["c1"]
    keys, vals = W.build_set(cfg)
    o = ArtOracle(keys, vals)
    q = W.lookup_batch(cfg, keys, 0, 100_003)
    ref = o.lookup(q)
    for t in (1, 3, 8):
        assert np.array_equal(o.lookup_mt(q, t), ref)
    assert np.array_equal(ref, MapOracle(keys, vals).lookup(q))


# ------------------------------------------------------------------ errors
def test_rejects_invalid():
    o = ArtOracle()
    assert o.insert_one(b"ab\x00", 1) == 0
    assert o.insert_one(b"ab", 2) == 1            # prefix of a stored key
    assert o.insert_one(b"ab\x00z", 2) == 1       # stored key is a prefix of it
    assert o.insert_one(b"", 3) == 2
    assert o.insert_one(b"x" * 33, 3) == 2
    assert o.insert_one(b"q\x00", MISS) == 3
    assert o.lookup_one(b"ab\x00") == 1
    # duplicates in build: last occurrence wins (reading C6)
    o2 = ArtOracle(np.array([5, 6, 5], dtype=np.uint64), np.array([1, 2, 3], dtype=np.uint64))
    assert o2.lookup(np.array([5, 6], dtype=np.uint64)).tolist() == [3, 2]
    m2 = MapOracle(np.array([5, 6, 5], dtype=np.uint64), np.array([1, 2, 3], dtype=np.uint64))
    assert m2.lookup(np.array([5, 6, 7], dtype=np.uint64)).tolist() == [3, 2, MISS]


# ------------------------------------------------------------------ map oracle vs ART oracle
def test_map_vs_art_on_c1_workload():
    import workloads as W
    cfg = W.CONFIGS["c1"]
    keys, vals = W.build_set(cfg)
    art = ArtOracle(keys, vals)
    mp = MapOracle(keys, vals)
    q = W.lookup_batch(cfg, keys, 0, 200_000)
    a = art.lookup(q)
    assert np.array_equal(a, mp.lookup(q))
    hit = a != OART_MISS
    assert abs(hit.mean() - 0.5) < 0.01         # 50% hit recipe
    # brute force on a sample: dict
    ref = dict(zip(keys.tolist(), vals.tolist()))
    for i in range(0, 200_000, 997):
        assert int(a[i]) == ref.get(int(q[i]), MISS)
    uk, uv = W.update_batch(cfg, keys)
    art.update(uk, uv)
    mp.update(uk, uv)
    for k, v in zip(uk.tolist(), uv.tolist()):
        if k in ref:
            ref[k] = v
    ak = art.lookup(keys)
    assert np.array_equal(ak, mp.lookup(keys))
    assert ak.tolist() == [ref[k] for k in keys.tolist()]
    st = art.stats()
    # c1 shape: 1 + 256 N256 at depths 0-1, then mostly N4
    assert st["n256"] == 257 and st["leaves"] == 65_536 and st["n4"] > 15_000


def test_map_oracle_strings_length_matters():
    slots = np.zeros((2, 32), np.uint8)
    slots[0, :3] = [97, 98, 0]
    slots[1, :2] = [97, 0]
    lens = np.array([3, 2], np.uint8)
    m = MapOracle((slots, lens), np.array([1, 2], np.uint64))
    q = np.zeros((3, 32), np.uint8)
    q[0, :3] = [97, 98, 0]
    q[1, :2] = [97, 98]
    q[2, :2] = [97, 0]
    assert m.lookup((q, np.array([3, 2, 2], np.uint8))).tolist() == [1, MISS, 2]


# ------------------------------------------------------------------ deletes (f1, P:137 / P:143)
def _k(x):
    return np.array(x, dtype=np.uint64)


def test_delete_hand_pins():
    keys = _k([1 << 40, 2 << 40, 3 << 40, 3 << 40 | 1])
    for O in (ArtOracle, MapOracle):
        o = O(keys, _k([10, 20, 30, 40]))
        # plain delete; delete of an absent key is a no-op
        o.apply(_k([keys[0], 12345]), None, [1, 1])
        assert o.lookup(keys).tolist() == [MISS, 20, 30, 40]
        # [delete k, update k] -> the higher index (the update) decides (reading C17)
        o.apply(_k([keys[1], keys[1]]), _k([0, 21]), [1, 0])
        # [update k, delete k] -> removed
        o.apply(_k([keys[2], keys[2]]), _k([31, 0]), [0, 1])
        assert o.lookup(keys).tolist() == [MISS, 21, MISS, 40]
        # a deleted key stays deleted: later updates are no-ops (no inserts on the device)
        o.apply(_k([keys[0], keys[2]]), _k([5, 6]), [0, 0])
        assert o.lookup(keys).tolist() == [MISS, 21, MISS, 40]


def test_delete_is_non_structural():
    """nodes are not collapsed.  Keys {x0, x1} under a 2-child N4 next to a
    leaf: deleting x1 leaves an N4 with ONE child (no path re-compression)."""
    keys = _k([0x0100000000000001, 0x0100000000000002, 0x0200000000000000])
    o = ArtOracle(keys, _k([1, 2, 3]))
    before = o.dump_structure().tolist()
    assert before[:5] == [1, 0, 2, 1, 2]
    assert o.erase_one((0x0100000000000002).to_bytes(8, "big")) == 1
    rec = o.dump_structure().tolist()
    # root N4 (2 children) -> child 0x01: N4, prefix 6 zero bytes, now one child
    assert rec[:5] == [1, 0, 2, 1, 2]
    assert rec[5:7] == [1, 6] and rec[13:15] == [1, 1]
    assert o.lookup(keys).tolist() == [1, MISS, 3]
    assert o.erase_one((0x0100000000000002).to_bytes(8, "big")) == 0


@pytest.mark.parametrize("seed", range(6))
def test_delete_batches_vs_bruteforce(seed):
    rng = random.Random(500 + seed)
    keys = _random_keyset(rng, 400, ["u64", "u64_shared", "bytes"][seed % 3])
    ref = {k: rng.getrandbits(62) for k in keys}
    o = ArtOracle()
    for k, v in ref.items():
        o.insert_one(k, v)
    mp = MapOracle(_as_input("bytes", keys), np.array([ref[k] for k in keys], np.uint64)) if seed % 3 == 2 else \
        MapOracle(_as_input("u64", keys), np.array([ref[k] for k in keys], np.uint64))
    for _ in range(4):
        ops = []
        for _ in range(600):
            k = rng.choice(keys) if rng.random() < 0.85 else bytes(rng.getrandbits(8) for _ in range(len(keys[0])))
            ops.append((k, rng.getrandbits(62), rng.random() < 0.3))
        # brute force, reading C17: presence before the batch, last op per present key decides
        present = set(ref)
        last = {}
        for k, v, d in ops:
            if k in present:
                last[k] = (v, d)
        for k, (v, d) in last.items():
            if d:
                del ref[k]
            else:
                ref[k] = v
        kind = "bytes" if seed % 3 == 2 else "u64"
        if kind == "u64" and any(len(k) != 8 for k, _, _ in ops):
            ops = [(k, v, d) for k, v, d in ops if len(k) == 8]
        inp = _as_input(kind, [k for k, _, _ in ops])
        vals = np.array([v for _, v, _ in ops], np.uint64)
        dele = np.array([d for _, _, d in ops], np.uint8)
        o.apply(inp, vals, dele)
        mp.apply(inp, vals, dele)
        q = _as_input(kind, keys)
        exp = [ref.get(k, MISS) for k in keys]
        assert o.lookup(q).tolist() == exp
        assert mp.lookup(q).tolist() == exp
        assert len(o) == len(ref)
        ks, ls, vs = o.dump_inorder()
        assert [(bytes(ks[i, : ls[i]]), int(vs[i])) for i in range(len(ls))] == sorted(ref.items())
