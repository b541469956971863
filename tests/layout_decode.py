"""Test-side decoder of the CuART flat layout.

Independent reading of the layout spec used to turn a host layout or a device
dump into the oracle's pre-order structure records, so builder/device results
can be compared with the oracle's pointer ART structure.
"""
from __future__ import annotations

import numpy as np

REC = {1: 64, 2: 160, 3: 672, 4: 2080, 5: 32, 6: 32, 7: 48}   # fallback; dumps carry record_bytes
VALOFF = {5: 8, 6: 16, 7: 32}
IDX_MASK = (1 << 52) - 1
HDR = {1: 40, 2: 0, 3: 0, 4: 0}   # header offset inside the record (N4 keeps keys + 3 children first)


def split_link(link: int):
    return link >> 60, (link >> 52) & 0xFF, link & IDX_MASK


def _u64(buf, off):
    return int(np.frombuffer(bytes(buf[off: off + 8]), dtype="<u8")[0])


MISS = (1 << 64) - 1


def _rec(view, t):
    return int(view["record_bytes"][t]) if "record_bytes" in view else REC[t]


def children(view, t, idx, live_only=True):
    """[(byte, child_link)] in byte order; deleted children (null link, or a leaf
    holding the tombstone value) are dropped unless live_only is False."""
    kids = _children_raw(view, t, idx)
    if not live_only:
        return kids
    return [(k, c) for k, c in kids if not (split_link(c)[0] >= 5 and leaf(view, c)[1] == MISS)]


def _children_raw(view, t, idx):
    b = view["buf"][t]
    o = idx * _rec(view, t)
    if t == 1 or t == 2:
        cnt = int(b[o + HDR[t] + 1]) + 1
        ko, co = (0, 8) if t == 1 else (16, 32)
        kids = [(int(b[o + ko + j]), _u64(b, o + co + 8 * j)) for j in range(cnt)]
        return [(k, c) for k, c in kids if c]
    if t == 3:
        out = []
        for byte in range(256):
            s = int(b[o + 16 + byte])
            if s != 0xFF and _u64(b, o + 272 + 8 * s):
                out.append((byte, _u64(b, o + 272 + 8 * s)))
        return out
    out = []
    for byte in range(256):
        c = _u64(b, o + 16 + 8 * byte)
        if c:
            out.append((byte, c))
    return out


def leaf(view, link):
    t, ln, idx = split_link(link)
    b = view["buf"][t]
    o = idx * _rec(view, t)
    return bytes(b[o: o + ln]), _u64(b, o + VALOFF[t]), bytes(b[o + ln: o + {5: 8, 6: 16, 7: 32}[t]])


def to_records(view) -> list[int]:
    """Pre-order records in the oracle dump format; asserts layout-internal consistency."""
    out: list[int] = []

    def first_leaf(link):
        while split_link(link)[0] < 5:
            t, _, idx = split_link(link)
            kids = children(view, t, idx, live_only=False)
            if not kids:
                return None
            link = kids[0][1]
        return leaf(view, link)[0]

    def rec(link, depth):
        t, aux, idx = split_link(link)
        assert t != 0
        if t >= 5:
            k, v, pad = leaf(view, link)
            assert pad == b"\0" * len(pad), "leaf key padding must be zero"
            assert t == (5 if len(k) <= 8 else 6 if len(k) <= 16 else 7), "leaf class by key length (P:110)"
            out.extend([0, len(k), *k, v - (1 << 64) if v >= 1 << 63 else v])   # oracle dumps int64
            return
        b = view["buf"][t]
        o = idx * _rec(view, t)
        h = o + HDR[t]
        plen = int(b[h])
        assert aux == depth + plen, "branch depth in the link = depth + prefix length"
        kids = children(view, t, idx)
        assert int(b[h + 1]) + 1 >= len(kids), "header count (deletes only remove children)"
        stored = bytes(b[h + 2: h + 2 + min(plen, 14)])
        fl = first_leaf(link)
        if fl is None:
            assert plen <= 14
            prefix = stored
        else:
            prefix = fl[depth: depth + plen]
        assert stored == prefix[:14], "header stores the first 14 prefix bytes"
        out.extend([t, plen, *prefix, len(kids), *[k for k, _ in kids]])
        for _, c in kids:
            rec(c, depth + plen + 1)

    root = view["root"]
    if root and not (split_link(root)[0] >= 5 and leaf(view, root)[1] == MISS):
        rec(root, 0)
    return out
