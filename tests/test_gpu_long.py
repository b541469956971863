"""§8(f) f4 — keys longer than 32 bytes (§3.2.3 option 2): inner nodes and
short-key leaves on the device, leaves of keys > 32 B in a host leaf buffer; the
GPU walk signals "compare on the host" at a host-leaf link and the library
finishes the compare.  Results must equal the plain-map oracle bit
for bit, for lookups and for update batches with duplicates."""
import numpy as np
import pytest

import paper_conf_icpp_koppehelggp21_b200 as C
from oracle import MapOracle, OART_MISS

pytestmark = pytest.mark.gpu
STRIDE = 256


def _slots(keys):
    """list of bytes -> the oracle's (slots[n, 256], lens) form."""
    slots = np.zeros((len(keys), STRIDE), np.uint8)
    lens = np.zeros(len(keys), np.uint8)
    for i, k in enumerate(keys):
        slots[i, : len(k)] = np.frombuffer(k, np.uint8)
        lens[i] = len(k)
    return slots, lens


def _keyset(rng, n, long_frac):
    """Prefix-free keys: content bytes in 1..255 plus a 0x00 terminator (reading C3).
    A `long_frac` share is 33..255 bytes, many of them sharing 40-byte prefixes in
    groups (deep paths below the 32-byte mark); the rest 1..32 bytes."""
    keys = set()
    stems = [bytes(rng.integers(1, 256, 40, dtype=np.uint8)) for _ in range(max(1, n // 64))]
    while len(keys) < n:
        if rng.random() < long_frac:
            l = int(rng.integers(33, 256))
            if rng.random() < 0.5:
                k = stems[int(rng.integers(0, len(stems)))] + bytes(rng.integers(1, 256, max(0, l - 41), dtype=np.uint8))
            else:
                k = bytes(rng.integers(1, 256, l - 1, dtype=np.uint8))
        else:
            l = int(rng.integers(1, 33))
            k = bytes(rng.integers(1, 256, l - 1, dtype=np.uint8))
        keys.add(k + b"\x00")
    return sorted(keys, key=lambda k: rng.random())


@pytest.mark.parametrize("long_frac", [0.03, 0.5])
@pytest.mark.parametrize("lut", [0, 2])
def test_long_keys_lookup_update(long_frac, lut):
    rng = np.random.default_rng(int(long_frac * 100) + lut)
    keys = _keyset(rng, 20_000, long_frac)
    assert max(len(k) for k in keys) > 32
    vals = rng.integers(0, 2**63, len(keys), dtype=np.uint64)
    ix = C.LongIndex(keys, vals, lut_bytes=lut)
    mp = MapOracle(_slots(keys), vals)
    # queries: hits; absent keys; a stored long key with its last content byte changed (the
    # walk reaches the host leaf, the host compare rejects); truncations (length differs)
    hits = [keys[int(i)] for i in rng.integers(0, len(keys), 30_000)]
    fresh = _keyset(np.random.default_rng(99), 5_000, long_frac)
    near = [k[:-2] + bytes([(k[-2] % 255) + 1]) + b"\x00" for k in hits[:5000] if len(k) > 33]
    trunc = [k[: len(k) // 2] for k in hits[:5000] if len(k) > 2]
    q = hits + fresh + near + trunc
    got = ix.lookup(q)
    exp = mp.lookup(_slots(q))
    assert np.array_equal(got, exp)
    assert (got[: len(hits)] != OART_MISS).all()
    # updates with many duplicates (last op wins) and absent keys (no-ops)
    uk = [keys[int(i)] for i in rng.integers(0, min(len(keys), 2000), 50_000)] + fresh[:1000]
    uv = rng.integers(0, 2**63, len(uk), dtype=np.uint64)
    ix.update(uk, uv)
    mp.update(_slots(uk), uv)
    allq = keys + fresh[:1000]
    assert np.array_equal(ix.lookup(allq), mp.lookup(_slots(allq)))
    ix.close()


def test_long_keys_errors():
    with pytest.raises(C.CuartError) as e:
        C.LongIndex([b"ab\x00", b"ab\x00cd"], np.array([1, 2], np.uint64))
    assert e.value.status == 3                                   # not prefix-free
    with pytest.raises(C.CuartError) as e:
        C.LongIndex([b"x" * 256], np.array([1], np.uint64))
    assert e.value.status == 2                                   # longer than 255
    ix = C.LongIndex([b"a" * 100 + b"\x00", b"b\x00"], np.array([7, 8], np.uint64))
    assert ix.lookup([b"a" * 100 + b"\x00", b"b\x00", b"c\x00"]).tolist() == [7, 8, int(OART_MISS)]
    with pytest.raises(C.CuartError):
        ix.lookup([b""])                                          # length 0
    ix.close()
