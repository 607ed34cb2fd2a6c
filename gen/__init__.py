"""Seeded synthetic corpus generator (shared input module for tests, smoke and bench).

Holds none of the indexing method's arithmetic: it only produces document bytes and
document offsets (``doc_off[i]..doc_off[i+1]`` is document ``i``).  The C++ source is
``gen/wjgen.cpp``; the recipe is documented there and in DESIGN.md ("Input recipe").

Workload configs follow BASELINE.json ``configs`` and SURVEY.md §8(d):

====  =====================  ========================================================
cfg   shape                  recipe
====  =====================  ========================================================
1     tiny                   1,000 docs, uniform [500,1500] B, Zipf V=10K, seed 1
2     ClueWeb09-shaped       1 GiB, lognormal mean 20 KB sigma 1.0, V=5M, seed 2
3     Wikipedia-shaped       4 x 1 GiB chunks, lognormal mean 3 KB sigma 0.8, V=2M
4     Library-of-Congress    8 x 1 GiB, lognormal mean 64 KB sigma 1.2, V=5M, 1% hapax
5     ClueWeb scale          64 x 1 GiB chunks, as config 2, seed 5
====  =====================  ========================================================
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, replace

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libwjgen.so")
_lib = None


class _Params(ctypes.Structure):
    _fields_ = [
        ("seed", ctypes.c_uint64),
        ("chunk", ctypes.c_uint64),
        ("n_docs", ctypes.c_uint64),
        ("target_bytes", ctypes.c_uint64),
        ("len_dist", ctypes.c_uint32),
        ("vocab", ctypes.c_uint32),
        ("len_mean", ctypes.c_double),
        ("len_sigma", ctypes.c_double),
        ("len_lo", ctypes.c_uint64),
        ("len_hi", ctypes.c_uint64),
        ("hapax_per100k", ctypes.c_uint32),
        ("long_permille", ctypes.c_uint32),
        ("threads", ctypes.c_uint32),
        ("reserved", ctypes.c_uint32),
    ]


def build(force: bool = False) -> str:
    """Compile gen/wjgen.cpp into gen/libwjgen.so (g++, no CUDA)."""
    src = os.path.join(_HERE, "wjgen.cpp")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        import subprocess

        subprocess.check_call(
            ["g++", "-O2", "-ffp-contract=off", "-fPIC", "-shared", "-pthread", "-o", _LIB_PATH, src]
        )
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        P = ctypes.POINTER
        lib.wjgen_layout.argtypes = [P(_Params), ctypes.c_void_p, ctypes.c_uint64, P(ctypes.c_uint64), P(ctypes.c_uint64)]
        lib.wjgen_layout.restype = ctypes.c_int
        lib.wjgen_fill.argtypes = [P(_Params), ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p]
        lib.wjgen_fill.restype = ctypes.c_int
        lib.wjgen_closed_form.argtypes = [ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p, P(ctypes.c_uint64)]
        lib.wjgen_closed_form.restype = ctypes.c_int
        _lib = lib
    return _lib


@dataclass(frozen=True)
class CorpusConfig:
    name: str
    seed: int
    chunks: int = 1
    n_docs: int = 0            # exact doc count (if > 0)
    chunk_bytes: int = 0       # else: bytes per chunk
    len_dist: int = 1          # 0 uniform, 1 lognormal
    len_mean: float = 20000.0
    len_sigma: float = 1.0
    len_lo: int = 64
    len_hi: int = 1 << 20
    vocab: int = 5_000_000
    hapax_per100k: int = 0
    long_permille: int = 1

    def scaled(self, chunk_bytes: int | None = None, chunks: int | None = None, vocab: int | None = None):
        kw = {}
        if chunk_bytes is not None:
            kw.update(chunk_bytes=int(chunk_bytes), n_docs=0)
        if chunks is not None:
            kw["chunks"] = int(chunks)
        if vocab is not None:
            kw["vocab"] = int(vocab)
        return replace(self, **kw)


GIB = 1 << 30
CONFIGS = {
    1: CorpusConfig("tiny", seed=1, n_docs=1000, len_dist=0, len_lo=500, len_hi=1500, vocab=10_000),
    2: CorpusConfig("clueweb", seed=2, chunk_bytes=GIB, len_mean=20000, len_sigma=1.0, vocab=5_000_000),
    3: CorpusConfig("wikipedia", seed=3, chunks=4, chunk_bytes=GIB, len_mean=3000, len_sigma=0.8, vocab=2_000_000),
    4: CorpusConfig("loc", seed=4, chunks=8, chunk_bytes=GIB, len_mean=65536, len_sigma=1.2,
                    len_hi=16 << 20, vocab=5_000_000, hapax_per100k=1000),
    5: CorpusConfig("clueweb-scale", seed=5, chunks=64, chunk_bytes=GIB, len_mean=20000, len_sigma=1.0, vocab=5_000_000),
}


def _params(cfg: CorpusConfig, chunk: int, threads: int = 0) -> _Params:
    return _Params(
        seed=cfg.seed, chunk=chunk, n_docs=cfg.n_docs, target_bytes=cfg.chunk_bytes,
        len_dist=cfg.len_dist, vocab=cfg.vocab, len_mean=cfg.len_mean, len_sigma=cfg.len_sigma,
        len_lo=cfg.len_lo, len_hi=cfg.len_hi, hapax_per100k=cfg.hapax_per100k,
        long_permille=cfg.long_permille, threads=threads, reserved=0,
    )


def layout(cfg: CorpusConfig, chunk: int = 0) -> np.ndarray:
    """Document offsets (u64, n_docs+1) of one chunk, without generating text."""
    lib = _load()
    p = _params(cfg, chunk)
    nd, nb = ctypes.c_uint64(), ctypes.c_uint64()
    if lib.wjgen_layout(ctypes.byref(p), None, 0, ctypes.byref(nd), ctypes.byref(nb)) != 0:
        raise RuntimeError("wjgen_layout sizing failed")
    doc_off = np.empty(nd.value + 1, dtype=np.uint64)
    if lib.wjgen_layout(ctypes.byref(p), doc_off.ctypes.data, doc_off.size, ctypes.byref(nd), ctypes.byref(nb)) != 0:
        raise RuntimeError("wjgen_layout failed")
    return doc_off


def fill(cfg: CorpusConfig, chunk: int, doc_off: np.ndarray, text_ptr: int, threads: int = 0) -> None:
    """Generate the chunk's text into caller memory at ``text_ptr`` (host, >= doc_off[-1] bytes)."""
    lib = _load()
    p = _params(cfg, chunk, threads)
    doc_off = np.ascontiguousarray(doc_off, dtype=np.uint64)
    if lib.wjgen_fill(ctypes.byref(p), doc_off.ctypes.data, doc_off.size - 1, ctypes.c_void_p(text_ptr)) != 0:
        raise RuntimeError("wjgen_fill failed")


def generate(cfg: CorpusConfig, chunk: int = 0, threads: int = 0):
    """Return (text: np.uint8[n_bytes], doc_off: np.uint64[n_docs+1]) for one chunk."""
    doc_off = layout(cfg, chunk)
    text = np.empty(int(doc_off[-1]), dtype=np.uint8)
    if text.size:
        fill(cfg, chunk, doc_off, text.ctypes.data, threads)
    return text, doc_off


def closed_form(n_docs: int, n_terms: int):
    """SURVEY.md §8(c) closed-form corpus: (text, doc_off)."""
    lib = _load()
    nb = ctypes.c_uint64()
    lib.wjgen_closed_form(n_docs, n_terms, None, None, ctypes.byref(nb))
    text = np.empty(nb.value, dtype=np.uint8)
    doc_off = np.empty(n_docs + 1, dtype=np.uint64)
    lib.wjgen_closed_form(n_docs, n_terms, ctypes.c_void_p(text.ctypes.data), ctypes.c_void_p(doc_off.ctypes.data), ctypes.byref(nb))
    return text, doc_off


def closed_form_term(j: int) -> bytes:
    code = (j * 7919 + 12345) % (26 ** 5)
    w = []
    for _ in range(5):
        w.append(chr(ord("a") + code % 26))
        code //= 26
    return "".join(reversed(w)).encode()


def from_docs(docs) -> tuple[np.ndarray, np.ndarray]:
    """Pack a list of byte strings into (text, doc_off)."""
    docs = [d.encode() if isinstance(d, str) else bytes(d) for d in docs]
    doc_off = np.zeros(len(docs) + 1, dtype=np.uint64)
    np.cumsum([len(d) for d in docs], out=doc_off[1:]) if docs else None
    text = np.frombuffer(b"".join(docs), dtype=np.uint8).copy()
    return text, doc_off


# English-like words for the parser Steps 3-4 tests: stems joined with the suffixes
# Porter's rules act on, plus the stop list's words, so stemming and stop-word removal fire often.
# Input generation only: nothing here stems or tests a word.
SUFFIXES = ["", "s", "es", "ies", "sses", "ss", "ed", "eed", "ing", "y", "ational", "tional", "enci", "anci",
            "izer", "abli", "alli", "entli", "eli", "ousli", "ization", "ation", "ator", "alism", "iveness",
            "fulness", "ousness", "aliti", "iviti", "biliti", "icate", "ative", "alize", "iciti", "ical", "ful",
            "ness", "al", "ance", "ence", "er", "ic", "able", "ible", "ant", "ement", "ment", "ent", "ion", "sion",
            "tion", "ou", "ism", "ate", "iti", "ous", "ive", "ize", "e", "ll", "led", "ling", "ings", "ers",
            "ations", "izing", "ally", "fully", "lessness", "ying", "yed"]
STEMS = ["relat", "condit", "ration", "valen", "hesit", "digit", "conform", "radic", "differ", "vil", "analog",
         "vietnam", "predic", "oper", "feud", "decis", "hope", "callous", "form", "sensit", "sensib", "trip",
         "electr", "good", "reviv", "allow", "infer", "airlin", "gyroscop", "adjust", "defens", "irrit",
         "replac", "depend", "adopt", "homolog", "commun", "activ", "angular", "effect", "bowdler", "prob",
         "rat", "ceas", "control", "rol", "cat", "pony", "ti", "caress", "feed", "agre", "plaster", "bl",
         "motor", "s", "conflat", "troubl", "siz", "hop", "tann", "fall", "hiss", "fizz", "fail", "fil",
         "happ", "sk", "gener", "oscill", "y", "by", "sy", "ay", "oy", "boy", "tr", "fl", "abc", "xyz",
         "book", "run", "sit", "lov", "mak", "nation", "organ", "class", "car", "ward", "quiet", "stud"]


def suffix_rich_docs(seed: int, n_docs: int, words_per_doc=(0, 120), stop_words=None) -> list:
    """Seeded documents of stem+suffix words, stop words (if given), numbers and a few non-ASCII
    words, with random capitalisation and punctuation."""
    rng = np.random.default_rng(seed)
    stop_words = list(stop_words or [])
    docs = []
    for _ in range(n_docs):
        n = int(rng.integers(words_per_doc[0], words_per_doc[1] + 1))
        out = []
        for _ in range(n):
            r = rng.random()
            if r < 0.25 and stop_words:
                w = stop_words[int(rng.integers(len(stop_words)))]
            elif r < 0.90:
                w = STEMS[int(rng.integers(len(STEMS)))] + SUFFIXES[int(rng.integers(len(SUFFIXES)))]
            elif r < 0.95:
                w = str(int(rng.integers(0, 10 ** int(rng.integers(1, 6)))))
            else:
                w = "año" + SUFFIXES[int(rng.integers(len(SUFFIXES)))]
            c = rng.random()
            if c < 0.08:
                w = w[:1].upper() + w[1:]
            elif c < 0.1:
                w = w.upper()
            out.append(w + [" ", " ", " ", ", ", ". ", "\n"][int(rng.integers(6))])
        docs.append("".join(out).encode("utf-8"))
    return docs


def suffix_rich_words(seed: int, n: int) -> list:
    """n seeded lowercase stem+suffix words (plus short words, digits and non-ASCII ones)."""
    rng = np.random.default_rng(seed)
    out = []
    for _ in range(n):
        r = rng.random()
        if r < 0.8:
            w = STEMS[int(rng.integers(len(STEMS)))] + SUFFIXES[int(rng.integers(len(SUFFIXES)))]
            if rng.random() < 0.3:
                w = SUFFIXES[int(rng.integers(len(SUFFIXES)))] + w
        elif r < 0.9:
            w = "".join(chr(97 + int(x)) for x in rng.integers(0, 26, size=int(rng.integers(1, 14))))
        elif r < 0.95:
            w = "".join("aeiouy"[int(x)] if x < 6 else chr(97 + int(x)) for x in rng.integers(0, 26, size=int(rng.integers(1, 9))))
        else:
            w = str(int(rng.integers(0, 99999))) + ("x" if rng.random() < 0.5 else "")
        out.append(w.encode())
    return out
