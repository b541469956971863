"""Test-side, independent statements of what an ART over a key set must look like.

Nothing here is imported by the oracle or by the product; these are the pins the
oracle is checked against (and, through the oracle, the CUDA path):

* ``canonical_records`` — an independent construction of the canonical
  path-compressed, lazily-expanded ART [17] by recursive partitioning of the
  sorted key set (one inner node per maximal group of >= 2 keys sharing a
  prefix; the node branches at the first byte where the group's keys differ).
  This is a different algorithm from the oracle's insert-based build.
* ``check_invariants`` — ART invariants (SURVEY §8(c) "What pins each part").
* golden-tree helpers for tests/golden/*.json.
"""
from __future__ import annotations

import json
import os

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
TYPE_CODES = {"N4": 1, "N16": 2, "N48": 3, "N256": 4}   # 1=N4, 2=N16, 3=N48, 4=N256


def node_type_for(count: int) -> int:
    """Insert-only ART: type fixed by child count (grow when full at 4/16/48)."""
    assert 2 <= count <= 256
    if count <= 4:
        return 1
    if count <= 16:
        return 2
    if count <= 48:
        return 3
    return 4


def load_golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def golden_key(kind, s):
    if kind == "u64":
        return int(s, 16).to_bytes(8, "big")
    if kind == "u32":
        return int(s, 16).to_bytes(4, "big")
    return bytes.fromhex(s)


def golden_tree_records(tree) -> list[int]:
    """Pre-order record stream (oracle dump format) of a hand-written golden tree."""
    out = []
    if "leaf" in tree:
        kb = bytes.fromhex(tree["leaf"])
        out += [0, len(kb), *kb, tree["value"]]
        return out
    pre = bytes.fromhex(tree["prefix"])
    kids = sorted(tree["children"].items(), key=lambda kv: int(kv[0], 16))
    out += [TYPE_CODES[tree["type"]], len(pre), *pre, len(kids), *[int(k, 16) for k, _ in kids]]
    for _, sub in kids:
        out += golden_tree_records(sub)
    return out


def _lcp(a: bytes, b: bytes, start: int) -> int:
    p = 0
    while start + p < len(a) and start + p < len(b) and a[start + p] == b[start + p]:
        p += 1
    return p


def canonical_records(items: list[tuple[bytes, int]]) -> list[int]:
    """Canonical ART of a prefix-free key set, built by recursive partition.

    items: (key bytes, value) with distinct keys.  Returns the pre-order record
    stream in the oracle's dump format (children in byte order)."""
    items = sorted(items)
    if not items:
        return []
    out: list[int] = []

    def rec(lo, hi, depth):
        if hi - lo == 1:
            k, v = items[lo]
            out.extend([0, len(k), *k, v])
            return
        first, last = items[lo][0], items[hi - 1][0]
        p = _lcp(first, last, depth)          # sorted => lcp(first,last) = lcp of the whole group
        d = depth + p
        groups = []
        i = lo
        while i < hi:
            b = items[i][0][d]                # prefix-free => every key has a byte at d
            j = i
            while j < hi and items[j][0][d] == b:
                j += 1
            groups.append((b, i, j))
            i = j
        out.extend([node_type_for(len(groups)), p, *first[depth:d], len(groups), *[g[0] for g in groups]])
        for _, i0, j0 in groups:
            rec(i0, j0, d + 1)

    rec(0, len(items), 0)
    return out


def parse_records(rec) -> list[dict]:
    """Pre-order record stream -> list of nodes with depth info (for invariant checks)."""
    rec = [int(x) for x in rec]
    pos = 0
    nodes = []

    def parse(depth, path):
        nonlocal pos
        kind = rec[pos]
        if kind == 0:
            ln = rec[pos + 1]
            key = bytes(rec[pos + 2: pos + 2 + ln])
            val = rec[pos + 2 + ln] & 0xFFFFFFFFFFFFFFFF
            pos += 3 + ln
            nodes.append({"kind": 0, "depth": depth, "key": key, "value": val, "path": path})
            return [key]
        plen = rec[pos + 1]
        prefix = bytes(rec[pos + 2: pos + 2 + plen])
        cnt = rec[pos + 2 + plen]
        cb = rec[pos + 3 + plen: pos + 3 + plen + cnt]
        pos += 3 + plen + cnt
        node = {"kind": kind, "depth": depth, "prefix": prefix, "children": cb, "path": path}
        nodes.append(node)
        keys = []
        sub = []
        for b in cb:
            ks = parse(depth + plen + 1, path + prefix + bytes([b]))
            sub.append(ks)
            keys += ks
        node["subkeys"] = sub
        return keys

    if rec:
        parse(0, b"")
        assert pos == len(rec)
    return nodes


def check_invariants(rec, items: dict[bytes, int]):
    """SURVEY §8(c) invariants 1-5 and 7's precondition, plus content == items."""
    nodes = parse_records(rec)
    if not items:
        assert nodes == []
        return
    if len(items) == 1:
        assert len(nodes) == 1 and nodes[0]["kind"] == 0
    leaves = [n for n in nodes if n["kind"] == 0]
    assert {n["key"]: n["value"] for n in leaves} == items
    assert len(leaves) == len(items)
    inorder = [n["key"] for n in leaves]
    assert inorder == sorted(inorder), "leaves must be in lexicographic order (P:110)"
    for n in nodes:
        if n["kind"] == 0:
            # prefix consistency: the path bytes equal the key's bytes at those offsets
            assert n["key"][: len(n["path"])] == n["path"]
            continue
        cb = n["children"]
        assert len(cb) >= 2, "inner node with < 2 children"
        assert n["kind"] == node_type_for(len(cb)), "type <-> child count (4/16/48/256)"
        assert list(cb) == sorted(set(cb)), "child bytes strictly increasing"
        # lazy expansion: every child subtree that is a single key is a leaf, and
        # the node's prefix is exactly the group's common prefix after `depth`
        allk = [k for ks in n["subkeys"] for k in ks]
        d = n["depth"]
        lcp = min(_lcp(allk[0], k, d) for k in allk[1:])
        assert lcp == len(n["prefix"]), "prefix must be the maximal common prefix (path compression)"
        for k in allk:
            assert k[: d + len(n["prefix"])] == n["path"] + n["prefix"]
    return nodes
