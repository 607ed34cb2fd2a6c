"""B200-native inverted-file indexer (Wei & JaJa, IPDPS 2011) — thin Python binding.

Argument marshalling only: every step of the indexing path runs in the sm_100a kernels of
``libwjindex.so`` behind the C ABI in ``include/wjindex.h``.  There is no CPU fallback: if the
library or a CUDA device is missing, ``Index()`` raises.

Names follow the C ABI: ``add_stream`` (index_add_stream), ``finalize``, ``read_postings``,
``serialize``, ``stats``, ``reset``.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libwjindex.so")

WJ_OK, WJ_NOT_FOUND = 0, 1
ERRORS = {-1: "WJ_ERR_INVALID_ARG", -2: "WJ_ERR_STATE", -3: "WJ_ERR_CUDA", -4: "WJ_ERR_NCCL", -5: "WJ_ERR_OOM",
          -6: "WJ_ERR_CAPACITY", -7: "WJ_ERR_BUFFER_TOO_SMALL"}
WJ_FLAG_PROFILE = 1
PHASES = ["h2d", "tokenize", "unique", "probe", "insert", "rebuild", "stream", "lexrank", "sort", "postings",
          "dict", "exchange", "vbyte", "stem"]
KERNELS = ["tokenize_count", "tokenize_emit", "probe", "slot_to_tid", "map_rank", "sort_hist", "sort_scatter",
           "rle_emit", "copy_partials"]
N_COLLECTIONS = 17613

EXPORTS = ["index_init", "index_add_stream", "index_finalize", "index_read_postings", "index_serialize",
           "index_stats", "index_reset", "index_debug_tokens", "index_debug_btree", "index_nccl_unique_id",
           "index_loopback_create", "index_loopback_destroy", "index_merge_serialized", "index_owner_map",
           "index_balance_owners", "index_stop_words", "index_debug_stem",
           "index_last_error", "index_destroy"]
WJ_FLAG_LOOPBACK = 2
WJ_FLAG_VBYTE = 4
WJ_FLAG_HOST_PIPELINE = 8
WJ_FLAG_BALANCED_OWNERS = 16
WJ_FLAG_STEM = 32
WJ_FLAG_STOPWORDS = 64
WJ_FLAG_HOT_TERMS = 128
WJ_FLAG_GLOBAL_STREAM = 512


class WJError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"{ERRORS.get(code, code)}: {msg}")
        self.code = code


class Config(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("nccl_unique_id", ctypes.c_void_p), ("stream", ctypes.c_void_p),
                ("max_chunk_bytes", ctypes.c_uint64), ("flags", ctypes.c_uint32), ("reserved", ctypes.c_uint32),
                ("workspace", ctypes.c_void_p), ("workspace_bytes", ctypes.c_uint64)]


class Stats(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in
                ("n_docs", "n_tokens", "n_dropped", "n_terms", "n_postings", "n_term_bytes", "n_chunks",
                 "kernel_launches", "host_syncs", "unique_terms_last", "new_terms_last", "btree_nodes",
                 "btree_height_max", "exchange_bytes", "device_bytes", "stream_elems", "table_retries",
                 "hot_elems_saved")] + [("exchange_ms", ctypes.c_double)] + [
        ("phase_ms", ctypes.c_double * 16), ("phase_launches", ctypes.c_uint64 * 16),
        ("kernel_ms", ctypes.c_double * len(KERNELS)), ("kernel_count", ctypes.c_uint64 * len(KERNELS))]


NODE_DTYPE = np.dtype([("count", "<u4"), ("cache", "<u4", 31), ("leaf", "<u4"), ("str", "<u4", 31),
                       ("pad", "<u4"), ("post", "<u4", 31), ("child", "<u4", 32)])
assert NODE_DTYPE.itemsize == 512

_lib = None


def _nccl_hint():
    """Point the library's dlopen at the NCCL torch ships (only used when world > 1)."""
    if "WJ_NCCL_LIB" in os.environ:
        return
    try:
        import nvidia.nccl
        base = list(nvidia.nccl.__path__)[0]
        cand = os.path.join(base, "lib", "libnccl.so.2")
        if os.path.exists(cand):
            os.environ["WJ_NCCL_LIB"] = cand
    except Exception:
        pass


def load_library():
    """Load libwjindex.so (in-tree).  Raises if it is missing: there is no fallback."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build() (nvcc sm_100a)")
        _nccl_hint()
        lib = ctypes.CDLL(LIB_PATH)
        vp, u64, u32, i32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
        P64 = ctypes.POINTER(ctypes.c_uint64)
        lib.index_init.argtypes = [ctypes.POINTER(vp), ctypes.POINTER(Config)]
        lib.index_add_stream.argtypes = [vp, vp, u64, vp, u64]
        lib.index_finalize.argtypes = [vp]
        lib.index_read_postings.argtypes = [vp, ctypes.c_char_p, u32, vp, vp, u64, P64]
        lib.index_serialize.argtypes = [vp, vp, u64, P64]
        lib.index_stats.argtypes = [vp, ctypes.POINTER(Stats)]
        lib.index_reset.argtypes = [vp]
        lib.index_debug_tokens.argtypes = [vp, vp, u64, vp, u64, u32, vp, u64, P64]
        lib.index_debug_btree.argtypes = [vp, vp, u64, P64, vp, vp, u64, P64]
        lib.index_last_error.argtypes = [vp]
        lib.index_last_error.restype = ctypes.c_char_p
        lib.index_destroy.argtypes = [vp]
        lib.index_nccl_unique_id.argtypes = [vp]
        lib.index_loopback_create.argtypes = [ctypes.c_int32, ctypes.POINTER(vp)]
        lib.index_loopback_destroy.argtypes = [vp]
        lib.index_merge_serialized.argtypes = [ctypes.c_int32, ctypes.POINTER(ctypes.c_void_p), ctypes.POINTER(ctypes.c_uint64),
                                               vp, u64, P64]
        for f in EXPORTS:
            if f not in ("index_last_error", "index_destroy", "index_loopback_destroy", "index_stop_words"):
                getattr(lib, f).restype = i32
        lib.index_owner_map.argtypes = [vp, vp, u32]
        lib.index_balance_owners.argtypes = [vp, u32, ctypes.c_int32, vp]
        lib.index_destroy.restype = None
        lib.index_stop_words.argtypes = []
        lib.index_stop_words.restype = ctypes.c_char_p
        lib.index_debug_stem.argtypes = [ctypes.c_int32, vp, vp, u32, vp, vp]
        lib.index_loopback_destroy.restype = None
        _lib = lib
    return _lib


def _ptr_len(x, dtype):
    """(pointer, n_elems, keepalive) for a torch tensor (cuda or cpu) or array-like."""
    try:
        import torch
        if isinstance(x, torch.Tensor):
            if not x.is_contiguous():
                x = x.contiguous()
            return x.data_ptr(), x.numel(), x
    except ImportError:  # pragma: no cover
        pass
    a = np.ascontiguousarray(x, dtype=dtype)
    return a.ctypes.data, a.size, a


def _current_stream(device):
    try:
        import torch
        if torch.cuda.is_available():
            return ctypes.c_void_p(torch.cuda.current_stream(device).cuda_stream)
    except Exception:  # pragma: no cover
        pass
    return ctypes.c_void_p(0)


class Index:
    """One indexing context on one GPU (index_init .. index_destroy)."""

    def __init__(self, device: int = 0, stream=None, profile: bool = False, rank: int = 0, world: int = 1,
                 nccl_id: bytes | None = None, hub: "LoopbackHub | None" = None, own_stream: bool = False,
                 vbyte: bool = False, pipeline: bool = False, balanced: bool = False, stem: bool = False,
                 stop: bool = False, hot: bool = False, workspace=None, global_stream: bool = False):
        """world > 1: pass nccl_id (128 bytes from nccl_unique_id(), broadcast by the caller) or a
        LoopbackHub shared by `world` contexts of this process (one host thread each).
        vbyte: finalize also builds the d-gap + variable-byte postings code; serialize() then
        returns the compressed file WJINV002.
        pipeline: host chunks are copied on a copy stream while the previous one is indexed
        (Fig. 9); keep each host buffer unchanged until the next call returns.
        balanced: world > 1, owners of the trie collections from a sampled bin-packing.
        stem / stop: the parser's Steps 3-4 (reading S20): Porter (1980)
        stems and removal of the built-in stop words (stop_words()).
        hot: sampled hot terms merged per document in the tokenizer for every chunk of >= 64 KiB
        (opt-in).
        workspace: a CUDA torch tensor (any dtype) whose memory the library sub-allocates for all of
        its device state instead of calling cudaMalloc; keep it alive until close().
        global_stream: one GPU, sort one global (term, docID) stream at finalize instead of building
        per-run partial postings lists (same bytes)."""
        self._lib = load_library()
        flags = (WJ_FLAG_PROFILE if profile else 0) | (WJ_FLAG_LOOPBACK if hub is not None else 0) | (
            WJ_FLAG_VBYTE if vbyte else 0) | (WJ_FLAG_HOST_PIPELINE if pipeline else 0) | (
            WJ_FLAG_BALANCED_OWNERS if balanced else 0) | (WJ_FLAG_STEM if stem else 0) | (
            WJ_FLAG_STOPWORDS if stop else 0) | (WJ_FLAG_HOT_TERMS if hot else 0) | (
            WJ_FLAG_GLOBAL_STREAM if global_stream else 0)
        self._nid = ctypes.create_string_buffer(bytes(nccl_id), 128) if nccl_id is not None else None
        uid = hub._h if hub is not None else (ctypes.cast(self._nid, ctypes.c_void_p) if self._nid is not None else None)
        if own_stream:
            strm = ctypes.c_void_p(0)
        else:
            strm = stream if stream is not None else _current_stream(device)
        ws_ptr, ws_bytes = None, 0
        self._ws = workspace
        if workspace is not None:
            ws_ptr, ws_bytes = workspace.data_ptr(), workspace.numel() * workspace.element_size()
        cfg = Config(device=device, rank=rank, world=world, nccl_unique_id=uid, stream=strm,
                     max_chunk_bytes=0, flags=flags, reserved=0, workspace=ws_ptr, workspace_bytes=ws_bytes)
        h = ctypes.c_void_p()
        rc = self._lib.index_init(ctypes.byref(h), ctypes.byref(cfg))
        if rc != WJ_OK:
            raise WJError(rc, self._lib.index_last_error(None).decode())
        self._h = h
        self._keep = []

    def _check(self, rc):
        if rc < 0:
            raise WJError(rc, self._lib.index_last_error(self._h).decode())
        return rc

    def close(self):
        if getattr(self, "_h", None):
            self._lib.index_destroy(self._h)
            self._h = None

    def __del__(self):
        self.close()

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def add_stream(self, text, doc_off):
        """Append one chunk: text (u8) and doc_off (u64, n_docs+1); host or device buffers."""
        tp, tn, tk = _ptr_len(text, np.uint8)
        dp, dn, dk = _ptr_len(doc_off, np.uint64)
        # buffers must stay alive until the next call returns (stream-ordered; with pipeline=True
        # a host chunk is read by the copy engine until the following call has indexed it)
        self._keep = (self._keep + [tk, dk])[-4:]
        self._check(self._lib.index_add_stream(self._h, tp, tn, dp, dn - 1))

    def finalize(self):
        self._check(self._lib.index_finalize(self._h))
        self._keep = []

    def read_postings(self, term: bytes):
        n = ctypes.c_uint64()
        rc = self._lib.index_read_postings(self._h, term, len(term), None, None, 0, ctypes.byref(n))
        if rc != -7:  # WJ_ERR_BUFFER_TOO_SMALL is the expected answer of the sizing call
            self._check(rc)
        if rc == WJ_NOT_FOUND:
            return None
        d = np.empty(n.value, dtype=np.uint32)
        t = np.empty(n.value, dtype=np.uint32)
        if n.value:
            rc = self._check(self._lib.index_read_postings(self._h, term, len(term), d.ctypes.data, t.ctypes.data,
                                                           n.value, ctypes.byref(n)))
        return d, t

    def serialize(self) -> bytes:
        n = ctypes.c_uint64()
        self._check(self._lib.index_serialize(self._h, None, 0, ctypes.byref(n)))
        buf = np.empty(n.value, dtype=np.uint8)
        self._check(self._lib.index_serialize(self._h, buf.ctypes.data, n.value, ctypes.byref(n)))
        return buf.tobytes()

    def owner_map(self) -> np.ndarray:
        """Owner rank of every trie collection (b mod world, or the balanced map once built)."""
        out = np.empty(N_COLLECTIONS, dtype=np.uint32)
        self._check(self._lib.index_owner_map(self._h, out.ctypes.data, N_COLLECTIONS))
        return out

    def serialized_size(self) -> int:
        n = ctypes.c_uint64()
        self._check(self._lib.index_serialize(self._h, None, 0, ctypes.byref(n)))
        return n.value

    def serialize_into(self, ptr: int, cap: int) -> int:
        """Serialize into caller memory (e.g. a pinned torch tensor's data_ptr()); returns bytes."""
        n = ctypes.c_uint64()
        self._check(self._lib.index_serialize(self._h, ctypes.c_void_p(ptr), cap, ctypes.byref(n)))
        return n.value

    def stats(self) -> dict:
        s = Stats()
        self._check(self._lib.index_stats(self._h, ctypes.byref(s)))
        out = {name: getattr(s, name) for name, _ in Stats._fields_[:19]}
        out["phase_ms"] = {PHASES[i]: s.phase_ms[i] for i in range(len(PHASES))}
        out["phase_launches"] = {PHASES[i]: s.phase_launches[i] for i in range(len(PHASES))}
        out["kernel_ms"] = {KERNELS[i]: s.kernel_ms[i] for i in range(len(KERNELS))}
        out["kernel_count"] = {KERNELS[i]: s.kernel_count[i] for i in range(len(KERNELS))}
        return out

    def reset(self):
        self._check(self._lib.index_reset(self._h))
        self._keep = []

    def debug_tokens(self, text, doc_off, doc_base: int = 0):
        tp, tn, tk = _ptr_len(text, np.uint8)
        dp, dn, dk = _ptr_len(doc_off, np.uint64)
        n = ctypes.c_uint64()
        self._check(self._lib.index_debug_tokens(self._h, tp, tn, dp, dn - 1, doc_base, None, 0, ctypes.byref(n)))
        out = np.empty(n.value, dtype=np.uint8)
        if n.value:
            self._check(self._lib.index_debug_tokens(self._h, tp, tn, dp, dn - 1, doc_base, out.ctypes.data, n.value,
                                                     ctypes.byref(n)))
        raw = out.tobytes()
        res, p = [], 0
        while p < len(raw):
            doc = int.from_bytes(raw[p:p + 4], "little")
            b = int.from_bytes(raw[p + 4:p + 6], "little")
            ln = raw[p + 6]
            res.append((doc, b, raw[p + 7:p + 7 + ln]))
            p += 7 + ln
        return res

    def debug_btree(self):
        nn, na = ctypes.c_uint64(), ctypes.c_uint64()
        self._check(self._lib.index_debug_btree(self._h, None, 0, ctypes.byref(nn), None, None, 0, ctypes.byref(na)))
        nodes = np.zeros(nn.value, dtype=NODE_DTYPE)
        coll = np.zeros((N_COLLECTIONS, 3), dtype=np.uint32)
        arena = np.zeros(max(na.value, 1), dtype=np.uint8)
        self._check(self._lib.index_debug_btree(self._h, nodes.ctypes.data, nn.value, ctypes.byref(nn),
                                                coll.ctypes.data, arena.ctypes.data, na.value, ctypes.byref(na)))
        return nodes, coll, arena[: na.value]


class LoopbackHub:
    """In-process exchange for `world` rank contexts driven by `world` host threads (one GPU)."""

    def __init__(self, world: int):
        self._lib = load_library()
        h = ctypes.c_void_p()
        rc = self._lib.index_loopback_create(world, ctypes.byref(h))
        if rc != WJ_OK:
            raise WJError(rc, "index_loopback_create")
        self._h = h
        self.world = world

    def close(self):
        if getattr(self, "_h", None):
            self._lib.index_loopback_destroy(self._h)
            self._h = None

    def __del__(self):
        self.close()


def nccl_unique_id() -> bytes:
    lib = load_library()
    buf = ctypes.create_string_buffer(128)
    rc = lib.index_nccl_unique_id(buf)
    if rc != WJ_OK:
        raise WJError(rc, lib.index_last_error(None).decode())
    return buf.raw


def merge_serialized(slices) -> bytes:
    """Merge the per-rank serialized slices into the global canonical inverted file (host)."""
    lib = load_library()
    k = len(slices)
    arrs = [np.frombuffer(bytes(x), dtype=np.uint8) for x in slices]
    ptrs = (ctypes.c_void_p * k)(*[a.ctypes.data for a in arrs])
    sizes = (ctypes.c_uint64 * k)(*[a.size for a in arrs])
    n = ctypes.c_uint64()
    rc = lib.index_merge_serialized(k, ptrs, sizes, None, 0, ctypes.byref(n))
    if rc != WJ_OK:
        raise WJError(rc, lib.index_last_error(None).decode())
    out = np.empty(n.value, dtype=np.uint8)
    rc = lib.index_merge_serialized(k, ptrs, sizes, out.ctypes.data, n.value, ctypes.byref(n))
    if rc != WJ_OK:
        raise WJError(rc, lib.index_last_error(None).decode())
    return out.tobytes()


def balance_owners(counts, world: int) -> np.ndarray:
    """The balanced owner map's bin packing (host) for per-collection token counts."""
    c = np.ascontiguousarray(counts, dtype=np.uint64)
    out = np.empty(len(c), dtype=np.uint32)
    rc = load_library().index_balance_owners(c.ctypes.data, len(c), world, out.ctypes.data)
    if rc != WJ_OK:
        raise WJError(rc, "index_balance_owners")
    return out


def stop_words() -> list:
    """The library's built-in stop list (index_stop_words; parser Step 4)."""
    return load_library().index_stop_words().decode().split()


def debug_stem(words, device: int = 0) -> list:
    """Porter stems of folded words computed by the device stemmer (index_debug_stem)."""
    words = [bytes(w) for w in words]
    off = np.zeros(len(words) + 1, dtype=np.uint32)
    off[1:] = np.cumsum([len(w) for w in words])
    packed = np.frombuffer(b"".join(words) + b"\0", dtype=np.uint8)
    out = np.zeros(max(int(off[-1]), 1), dtype=np.uint8)
    lens = np.zeros(max(len(words), 1), dtype=np.uint32)
    rc = load_library().index_debug_stem(device, packed.ctypes.data, off.ctypes.data, len(words), out.ctypes.data,
                                         lens.ctypes.data)
    if rc != WJ_OK:
        raise WJError(rc, "index_debug_stem")
    raw = out.tobytes()
    return [raw[int(off[i]):int(off[i]) + int(lens[i])] for i in range(len(words))]


def owner_of(collection: int, world: int) -> int:
    """Rank owning a trie collection: index i goes to GPU i mod N_2."""
    return collection % world


def build_index(text, doc_off, device: int = 0, chunks=None) -> bytes:
    """Convenience: index documents (optionally as several add_stream chunks) and serialize."""
    with Index(device=device) as ix:
        if chunks is None:
            ix.add_stream(text, doc_off)
        else:
            off = np.asarray(doc_off, dtype=np.uint64)
            for a, b in chunks:
                ix.add_stream(np.asarray(text)[int(off[a]):int(off[b])], off[a:b + 1] - off[a])
        ix.finalize()
        return ix.serialize()
