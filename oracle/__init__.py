"""CPU oracle (TEST INFRASTRUCTURE ONLY).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_ipps_weij11_b200``) never imports it and has no CPU fallback.

The C++ source (``oracle/oracle.cpp``) is a plain ``std::map<std::string,
vector<(docID, tf)>>`` written from the paper's problem statement (PAPER.md P:35, P:39,
P:162) and Table I for the trie-collection index.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "oracle.cpp")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        subprocess.check_call(["g++", "-O2", "-fPIC", "-shared", "-pthread", "-o", _LIB_PATH, src])
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        vp, u64, u32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32
        P64 = ctypes.POINTER(ctypes.c_uint64)
        lib.oracle_bucket.argtypes = [ctypes.c_char_p, u32]
        lib.oracle_bucket.restype = ctypes.c_int
        lib.oracle_new.restype = vp
        lib.oracle_free.argtypes = [vp]
        lib.oracle_add.argtypes = [vp, vp, vp, u64]
        lib.oracle_add.restype = ctypes.c_int
        lib.oracle_add_mt.argtypes = [vp, vp, vp, u64, ctypes.c_int]
        lib.oracle_add_mt.restype = ctypes.c_int
        lib.oracle_serialize.argtypes = [vp, vp, u64, P64]
        lib.oracle_serialize.restype = ctypes.c_int
        lib.oracle_serialize_vbyte.argtypes = [vp, vp, u64, P64]
        lib.oracle_serialize_vbyte.restype = ctypes.c_int
        lib.oracle_vbyte.argtypes = [vp, u64, vp]
        lib.oracle_vbyte.restype = u64
        lib.oracle_set_options.argtypes = [vp, ctypes.c_int, ctypes.c_int]
        lib.oracle_set_options.restype = ctypes.c_int
        lib.oracle_porter.argtypes = [ctypes.c_char_p, u32, ctypes.c_int, vp]
        lib.oracle_porter.restype = ctypes.c_int
        lib.oracle_stop_words.restype = ctypes.c_char_p
        lib.oracle_postings.argtypes = [vp, ctypes.c_char_p, u32, vp, vp, u64, P64]
        lib.oracle_postings.restype = ctypes.c_int
        lib.oracle_dump_tokens.argtypes = [vp, vp, u64, u32, vp, u64, P64]
        lib.oracle_dump_tokens.restype = ctypes.c_int
        _lib = lib
    return _lib


def bucket(term: bytes) -> int:
    """Trie-collection index of a folded term (Table I)."""
    return _load().oracle_bucket(term, len(term))


class Oracle:
    """Incremental oracle: add() chunks of documents in submission order, then serialize()."""

    def __init__(self, stem: bool = False, stop: bool = False):
        """stem / stop: the parser's Steps 3-4 (reading S20)."""
        self._lib = _load()
        self._h = self._lib.oracle_new()
        if stem or stop:
            self._lib.oracle_set_options(self._h, int(stem), int(stop))

    def close(self):
        if self._h:
            self._lib.oracle_free(self._h)
            self._h = None

    def __del__(self):
        self.close()

    def add(self, text: np.ndarray, doc_off: np.ndarray, threads: int = 1) -> None:
        text = np.ascontiguousarray(text, dtype=np.uint8)
        doc_off = np.ascontiguousarray(doc_off, dtype=np.uint64)
        n_docs = doc_off.size - 1
        if threads > 1:
            rc = self._lib.oracle_add_mt(self._h, text.ctypes.data, doc_off.ctypes.data, n_docs, threads)
        else:
            rc = self._lib.oracle_add(self._h, text.ctypes.data, doc_off.ctypes.data, n_docs)
        if rc != 0:
            raise RuntimeError(f"oracle_add failed: {rc}")

    def serialize(self, vbyte: bool = False) -> bytes:
        """Canonical index bytes: WJINV001, or WJINV002 (d-gap + variable-byte postings) if vbyte."""
        f = self._lib.oracle_serialize_vbyte if vbyte else self._lib.oracle_serialize
        n = ctypes.c_uint64()
        f(self._h, None, 0, ctypes.byref(n))
        buf = ctypes.create_string_buffer(n.value)
        rc = f(self._h, buf, n.value, ctypes.byref(n))
        if rc != 0:
            raise RuntimeError(f"oracle_serialize failed: {rc}")
        return buf.raw[: n.value]

    def postings(self, term: bytes):
        n = ctypes.c_uint64()
        rc = self._lib.oracle_postings(self._h, term, len(term), None, None, 0, ctypes.byref(n))
        if rc == 1:
            return None
        d = np.empty(n.value, dtype=np.uint32)
        t = np.empty(n.value, dtype=np.uint32)
        rc = self._lib.oracle_postings(self._h, term, len(term), d.ctypes.data, t.ctypes.data, n.value, ctypes.byref(n))
        assert rc == 0
        return d, t


def index_bytes(text, doc_off, threads: int = 1, vbyte: bool = False, stem: bool = False,
                stop: bool = False) -> bytes:
    """Serialized oracle index of one batch of documents."""
    o = Oracle(stem, stop)
    o.add(text, doc_off, threads)
    return o.serialize(vbyte)


def porter(term: bytes, step: int = -1) -> bytes:
    """Porter (1980) stem of a folded term; step 0..7 applies only step 1a,1b,1c,2,3,4,5a,5b."""
    out = ctypes.create_string_buffer(len(term) + 1)
    n = _load().oracle_porter(term, len(term), step, out)
    return out.raw[:n]


def stop_words() -> list:
    """The oracle's stop list (parser Step 4)."""
    return _load().oracle_stop_words().decode().split()


def vbyte(values) -> bytes:
    """Variable-byte code of a sequence of u32 values (reading S19)."""
    v = np.ascontiguousarray(values, dtype=np.uint32)
    lib = _load()
    out = ctypes.create_string_buffer(5 * max(len(v), 1))
    n = lib.oracle_vbyte(v.ctypes.data, len(v), out)
    return out.raw[:n]


def dump_tokens(text, doc_off, doc_base: int = 0):
    """List of (docID, bucket, term bytes) for every kept token, in text order."""
    lib = _load()
    text = np.ascontiguousarray(text, dtype=np.uint8)
    doc_off = np.ascontiguousarray(doc_off, dtype=np.uint64)
    n = ctypes.c_uint64()
    lib.oracle_dump_tokens(text.ctypes.data, doc_off.ctypes.data, doc_off.size - 1, doc_base, None, 0, ctypes.byref(n))
    buf = np.empty(n.value, dtype=np.uint8)
    rc = lib.oracle_dump_tokens(text.ctypes.data, doc_off.ctypes.data, doc_off.size - 1, doc_base,
                                buf.ctypes.data, n.value, ctypes.byref(n))
    assert rc == 0
    out = []
    raw = buf.tobytes()
    p = 0
    while p < len(raw):
        doc = int.from_bytes(raw[p:p + 4], "little")
        b = int.from_bytes(raw[p + 4:p + 6], "little")
        ln = raw[p + 6]
        out.append((doc, b, raw[p + 7:p + 7 + ln]))
        p += 7 + ln
    return out
