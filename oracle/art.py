"""ctypes wrapper of oracle/art_oracle.c and the plain-definition MapOracle.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

OART_MISS = np.uint64(0xFFFFFFFFFFFFFFFF)
MAX_KEY = 32  # compile-time maximum key length
_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "art_oracle.c")
_LIB = os.path.join(_HERE, "liboart.so")
_lib = None


def build_oracle_lib(force: bool = False) -> str:
    """Compile art_oracle.c with plain gcc (no OpenMP, no vectorisation tricks)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-pthread", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build_oracle_lib())
        P, U64, U32, SZ = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_size_t
        lib.oart_new.restype = P
        lib.oart_free.argtypes = [P]
        lib.oart_insert.argtypes = [P, P, U32, U64]
        lib.oart_insert.restype = ctypes.c_int
        lib.oart_insert_batch.argtypes = [P, P, P, U32, SZ, P, SZ]
        lib.oart_insert_batch.restype = ctypes.c_int
        lib.oart_size.argtypes = [P]
        lib.oart_size.restype = U64
        lib.oart_lookup.argtypes = [P, P, U32]
        lib.oart_lookup.restype = U64
        lib.oart_lookup_batch.argtypes = [P, P, P, U32, SZ, SZ, P]
        lib.oart_lookup_batch_mt.argtypes = [P, P, P, U32, SZ, SZ, P, ctypes.c_int]
        lib.oart_lookup_batch_mt.restype = ctypes.c_int
        lib.oart_update_batch.argtypes = [P, P, P, U32, SZ, P, SZ, P]
        lib.oart_update_batch.restype = ctypes.c_int64
        lib.oart_dump_inorder.argtypes = [P, P, P, P, SZ]
        lib.oart_dump_inorder.restype = SZ
        lib.oart_dump_structure.argtypes = [P, P, SZ]
        lib.oart_dump_structure.restype = SZ
        lib.oart_stats.argtypes = [P, P]
        lib.oart_erase.argtypes = [P, P, U32]
        lib.oart_erase.restype = ctypes.c_int
        lib.oart_apply_batch.argtypes = [P, P, P, U32, SZ, P, P, SZ, P]
        lib.oart_apply_batch.restype = ctypes.c_int64
        _lib = lib
    return _lib


def canonical_bytes(keys, kind: str | None = None):
    """Key canonicalisation for the oracle (reading C2: integers are compared as
    big-endian byte strings, so lexicographic order = numeric order [17]).

    Returns (slots uint8[n, stride] C-contiguous, lens uint8[n] or None, fixed_len, stride).
    ``keys`` is a uint64/uint32 array, or a (slots uint8[n,32], lens uint8[n]) tuple.
    """
    if isinstance(keys, tuple):
        slots, lens = keys
        slots = np.ascontiguousarray(slots, dtype=np.uint8)
        lens = np.ascontiguousarray(lens, dtype=np.uint8)
        return slots, lens, 0, slots.shape[1]
    keys = np.asarray(keys)
    if keys.dtype == np.uint64:
        be = np.ascontiguousarray(keys.astype(">u8")).view(np.uint8).reshape(-1, 8)
        return be, None, 8, 8
    if keys.dtype == np.uint32:
        be = np.ascontiguousarray(keys.astype(">u4")).view(np.uint8).reshape(-1, 4)
        return be, None, 4, 4
    raise TypeError(f"unsupported key dtype {keys.dtype}")


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


class ArtOracle:
    """Plain pointer ART (Leis [17]); insert / lookup / sequential update / dumps."""

    def __init__(self, keys=None, values=None):
        self._lib = _load()
        self._t = self._lib.oart_new()
        if keys is not None:
            self.insert(keys, values)

    def close(self):
        if self._t:
            self._lib.oart_free(self._t)
            self._t = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __len__(self):
        return int(self._lib.oart_size(self._t))

    def insert(self, keys, values):
        slots, lens, flen, stride = canonical_bytes(keys)
        vals = np.ascontiguousarray(values, dtype=np.uint64)
        assert vals.shape[0] == slots.shape[0]
        rc = self._lib.oart_insert_batch(self._t, _ptr(slots), _ptr(lens), flen, stride, _ptr(vals), slots.shape[0])
        if rc == 1:
            raise ValueError("key set is not prefix-free")
        if rc == 2:
            raise ValueError("key length must be 1..32")
        if rc == 3:
            raise ValueError("value is the reserved miss value")

    def insert_one(self, key: bytes, value: int) -> int:
        buf = (ctypes.c_uint8 * max(1, len(key))).from_buffer_copy(key or b"\0")
        return self._lib.oart_insert(self._t, buf, len(key), value)

    def lookup_one(self, key: bytes) -> int:
        buf = (ctypes.c_uint8 * max(1, len(key))).from_buffer_copy(key or b"\0")
        return int(self._lib.oart_lookup(self._t, buf, len(key)))

    def lookup(self, queries) -> np.ndarray:
        slots, lens, flen, stride = canonical_bytes(queries)
        out = np.empty(slots.shape[0], dtype=np.uint64)
        self._lib.oart_lookup_batch(self._t, _ptr(slots), _ptr(lens), flen, stride, slots.shape[0], _ptr(out))
        return out

    def lookup_mt(self, queries, threads: int) -> np.ndarray:
        """oart_lookup_batch split over `threads` POSIX threads (read-only)."""
        slots, lens, flen, stride = canonical_bytes(queries)
        out = np.empty(slots.shape[0], dtype=np.uint64)
        self._lib.oart_lookup_batch_mt(self._t, _ptr(slots), _ptr(lens), flen, stride, slots.shape[0], _ptr(out),
                                       int(threads))
        return out

    def update(self, keys, values) -> int:
        """Sequential batch update; ops carrying the reserved value are dropped
        (reading C5) and counted in ``self.last_rejected``.  Returns the number of
        applied ops that hit a stored key."""
        slots, lens, flen, stride = canonical_bytes(keys)
        vals = np.ascontiguousarray(values, dtype=np.uint64)
        rej = ctypes.c_uint64()
        hits = self._lib.oart_update_batch(self._t, _ptr(slots), _ptr(lens), flen, stride, _ptr(vals), slots.shape[0],
                                           ctypes.byref(rej))
        self.last_rejected = int(rej.value)
        return int(hits)

    def erase_one(self, key: bytes) -> int:
        buf = (ctypes.c_uint8 * max(1, len(key))).from_buffer_copy(key or b"\0")
        return int(self._lib.oart_erase(self._t, buf, len(key)))

    def apply(self, keys, values, is_delete) -> int:
        """Batch of updates and deletes (reading C17: keys located on the pre-batch
        state, the highest op index per key decides: value, or removal)."""
        slots, lens, flen, stride = canonical_bytes(keys)
        n = slots.shape[0]
        vals = np.ascontiguousarray(values if values is not None else np.zeros(n), dtype=np.uint64)
        dele = np.ascontiguousarray(is_delete, dtype=np.uint8) if is_delete is not None else None
        rej = ctypes.c_uint64()
        hits = self._lib.oart_apply_batch(self._t, _ptr(slots), _ptr(lens), flen, stride, _ptr(vals), _ptr(dele), n,
                                          ctypes.byref(rej))
        self.last_rejected = int(rej.value)
        return int(hits)

    def dump_inorder(self):
        n = len(self)
        keys = np.zeros((n, MAX_KEY), dtype=np.uint8)
        lens = np.zeros(n, dtype=np.uint8)
        vals = np.zeros(n, dtype=np.uint64)
        got = self._lib.oart_dump_inorder(self._t, _ptr(keys), _ptr(lens), _ptr(vals), n)
        assert got == n
        return keys, lens, vals

    def dump_structure(self) -> np.ndarray:
        need = self._lib.oart_dump_structure(self._t, None, 0)
        buf = np.zeros(max(1, need), dtype=np.int64)
        self._lib.oart_dump_structure(self._t, _ptr(buf), need)
        return buf[:need]

    def stats(self) -> dict:
        out = np.zeros(6, dtype=np.uint64)
        self._lib.oart_stats(self._t, _ptr(out))
        return {"leaves": int(out[0]), "n4": int(out[1]), "n16": int(out[2]), "n48": int(out[3]),
                "n256": int(out[4]), "height": int(out[5])}


class MapOracle:
    """The plain definition: a finite map with sequential updates.

    Keys are held as canonical byte strings (zero-padded to ``stride`` bytes plus
    the true length), sorted lexicographically; lookup is a binary search
    (numpy.searchsorted on void-typed rows compares bytes lexicographically).
    """

    def __init__(self, keys, values):
        slots, lens, flen, stride = canonical_bytes(keys)
        self.stride = stride
        self.fixed = lens is None
        rows = self._rows(slots, lens, flen)
        vals = np.ascontiguousarray(values, dtype=np.uint64)
        # duplicates: last occurrence wins (reading C6) -> stable sort, keep last of each run
        order = np.argsort(rows, kind="stable")
        rows_s = rows[order]
        last = np.ones(rows_s.shape[0], dtype=bool)
        last[:-1] = rows_s[1:] != rows_s[:-1]
        self.rows = rows_s[last]
        self.values = vals[order][last].copy()
        self.present = np.ones(self.rows.shape[0], dtype=bool)

    def _rows(self, slots, lens, flen):
        if lens is None:
            # fixed-length keys: the big-endian bytes read as one unsigned integer
            # compare exactly like the byte strings (lexicographic = numeric order),
            # and numpy sorts / searches integers much faster than void rows
            if slots.shape[1] in (4, 8):
                be = ">u8" if slots.shape[1] == 8 else ">u4"
                return np.ascontiguousarray(slots).view(be).ravel().astype(be[1:])
            return np.ascontiguousarray(slots).view(np.dtype((np.void, slots.shape[1]))).ravel()
        # append the length byte AFTER the zero-padded content so "ab"(2) != "ab\0"(3);
        # for a prefix-free set this keeps lexicographic order of the true keys.
        ext = np.concatenate([slots, lens[:, None]], axis=1)
        return np.ascontiguousarray(ext).view(np.dtype((np.void, ext.shape[1]))).ravel()

    def _find(self, keys):
        slots, lens, flen, stride = canonical_bytes(keys)
        q = self._rows(slots, lens, flen)
        pos = np.searchsorted(self.rows, q)
        pos_c = np.minimum(pos, max(0, self.rows.shape[0] - 1))
        found = (pos < self.rows.shape[0]) & (self.rows[pos_c] == q) if self.rows.shape[0] else np.zeros(q.shape[0], bool)
        return pos_c, found

    def lookup(self, queries) -> np.ndarray:
        pos, found = self._find(queries)
        if found.shape[0]:
            found &= self.present[pos]
        out = np.full(found.shape[0], OART_MISS, dtype=np.uint64)
        out[found] = self.values[pos[found]]
        return out

    def update(self, keys, values) -> int:
        """Ops applied in index order; equivalently the highest op index per key
        wins.  Absent keys are no-ops (reading C6); ops carrying the
        reserved value are dropped (reading C5) and counted in last_rejected."""
        vals = np.ascontiguousarray(values, dtype=np.uint64)
        pos, found = self._find(keys)
        reserved = vals == OART_MISS
        self.last_rejected = int(reserved.sum())
        if found.shape[0]:
            found &= self.present[pos] & ~reserved
        idx = np.nonzero(found)[0]
        # sequential application == for each key, the value of its LAST op
        p = pos[idx]
        order = np.argsort(p, kind="stable")
        p_s, i_s = p[order], idx[order]
        last = np.ones(p_s.shape[0], dtype=bool)
        last[:-1] = p_s[1:] != p_s[:-1]
        self.values[p_s[last]] = vals[i_s[last]]
        return int(idx.shape[0])

    def apply(self, keys, values, is_delete) -> int:
        """Reading C17: presence is taken before the batch; per present key the op
        with the highest index decides (store its value, or remove the key)."""
        n = len(is_delete)
        vals = np.ascontiguousarray(values if values is not None else np.zeros(n), dtype=np.uint64)
        dele = np.asarray(is_delete, dtype=bool)
        pos, found = self._find(keys)
        reserved = ~dele & (vals == OART_MISS)          # reading C5: dropped
        self.last_rejected = int(reserved.sum())
        if found.shape[0]:
            found &= self.present[pos] & ~reserved
        idx = np.nonzero(found)[0]
        p = pos[idx]
        order = np.argsort(p, kind="stable")
        p_s, i_s = p[order], idx[order]
        last = np.ones(p_s.shape[0], dtype=bool)
        last[:-1] = p_s[1:] != p_s[:-1]
        wp, wi = p_s[last], i_s[last]
        d = dele[wi]
        self.values[wp[~d]] = vals[wi[~d]]
        self.present[wp[d]] = False
        return int(idx.shape[0])

    def items(self):
        return self.rows, self.values
