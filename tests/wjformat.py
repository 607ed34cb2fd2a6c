"""Reader + invariant checker for the canonical serialized inverted file.

Layout (little-endian):  64-B header {char magic[8]="WJINV001"; u64 n_docs, n_tokens,
n_dropped, n_terms, n_postings, n_term_bytes, reserved}; u64 term_off[n_terms+1];
u8 term_bytes[] (pad 8); u32 df[] (pad 8); u64 cf[]; u64 post_off[n_terms+1];
u32 docid[] (pad 8); u32 tf[] (pad 8).

Compressed layout "WJINV002" (reading S19): same header with word 7 =
n_post_bytes, same dictionary / df / cf; then u64 post_off[n_terms+1] as BYTE offsets and the
postings bytes (pad 8): per posting vbyte(d-gap) then vbyte(tf); vbyte = 7-bit groups, least
significant first, high bit set iff more bytes follow; the first gap of a list is the docID.
`parse` accepts both and returns the decoded (uncompressed) index.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

MAGIC = b"WJINV001"
MAGIC_VB = b"WJINV002"


def _pad8(n: int) -> int:
    return (n + 7) & ~7


@dataclass
class Index:
    n_docs: int
    n_tokens: int
    n_dropped: int
    n_terms: int
    n_postings: int
    n_term_bytes: int
    term_off: np.ndarray
    term_bytes: bytes
    df: np.ndarray
    cf: np.ndarray
    post_off: np.ndarray
    docid: np.ndarray
    tf: np.ndarray

    def term(self, i: int) -> bytes:
        return self.term_bytes[int(self.term_off[i]):int(self.term_off[i + 1])]

    def terms(self):
        return [self.term(i) for i in range(self.n_terms)]

    def postings(self, i: int):
        a, b = int(self.post_off[i]), int(self.post_off[i + 1])
        return self.docid[a:b], self.tf[a:b]

    def as_dict(self):
        out = {}
        for i in range(self.n_terms):
            d, t = self.postings(i)
            out[self.term(i)] = list(zip(d.tolist(), t.tolist()))
        return out


def vbyte_decode(code: bytes, n_values: int):
    """Decode n_values variable-byte values from code; returns (values, bytes consumed)."""
    out = []
    p = 0
    for _ in range(n_values):
        v = shift = 0
        while True:
            c = code[p]
            p += 1
            v |= (c & 0x7F) << shift
            shift += 7
            if not c & 0x80:
                break
        out.append(v)
    return out, p


def parse(buf: bytes) -> Index:
    vb = buf[:8] == MAGIC_VB
    if buf[:8] != MAGIC and not vb:
        raise ValueError("bad magic")
    hdr = np.frombuffer(buf, dtype="<u8", count=8)
    n_docs, n_tokens, n_dropped, n_terms, n_post, n_tb, reserved = (int(x) for x in hdr[1:8])
    if reserved != 0 and not vb:
        raise ValueError("reserved != 0")
    p = 64
    term_off = np.frombuffer(buf, dtype="<u8", count=n_terms + 1, offset=p); p += 8 * (n_terms + 1)
    term_bytes = buf[p:p + n_tb]
    if any(buf[p + n_tb:p + _pad8(n_tb)]):
        raise ValueError("nonzero padding after term bytes")
    p += _pad8(n_tb)
    df = np.frombuffer(buf, dtype="<u4", count=n_terms, offset=p); p += _pad8(4 * n_terms)
    cf = np.frombuffer(buf, dtype="<u8", count=n_terms, offset=p); p += 8 * n_terms
    post_off = np.frombuffer(buf, dtype="<u8", count=n_terms + 1, offset=p); p += 8 * (n_terms + 1)
    if vb:
        n_pb = reserved
        code = buf[p:p + n_pb]
        if any(buf[p + n_pb:p + _pad8(n_pb)]):
            raise ValueError("nonzero padding after postings bytes")
        p += _pad8(n_pb)
        if p != len(buf):
            raise ValueError(f"trailing bytes: parsed {p} of {len(buf)}")
        if post_off[0] != 0 or post_off[-1] != n_pb:
            raise ValueError("postings byte offsets do not span the code")
        docid = np.empty(n_post, dtype=np.uint32)
        tf = np.empty(n_post, dtype=np.uint32)
        k = 0
        for i in range(n_terms):
            a, b = int(post_off[i]), int(post_off[i + 1])
            vals, used = vbyte_decode(code[a:b], 2 * int(df[i]))
            if used != b - a:
                raise ValueError(f"term {i}: postings bytes not consumed exactly")
            gaps = np.array(vals[0::2], dtype=np.int64)
            docid[k:k + int(df[i])] = np.cumsum(gaps)
            tf[k:k + int(df[i])] = vals[1::2]
            k += int(df[i])
        if k != n_post:
            raise ValueError("sum df != n_postings")
        post_off = np.concatenate([[0], np.cumsum(df.astype(np.uint64))]).astype(np.uint64)
        return Index(n_docs, n_tokens, n_dropped, n_terms, n_post, n_tb, term_off, term_bytes, df, cf,
                     post_off, docid, tf)
    docid = np.frombuffer(buf, dtype="<u4", count=n_post, offset=p); p += _pad8(4 * n_post)
    tf = np.frombuffer(buf, dtype="<u4", count=n_post, offset=p); p += _pad8(4 * n_post)
    if p != len(buf):
        raise ValueError(f"trailing bytes: parsed {p} of {len(buf)}")
    return Index(n_docs, n_tokens, n_dropped, n_terms, n_post, n_tb, term_off, term_bytes, df, cf,
                 post_off, docid, tf)


def check_invariants(ix: Index) -> None:
    """SURVEY.md §8(c) invariants: raises AssertionError on violation."""
    assert ix.term_off[0] == 0 and ix.term_off[-1] == ix.n_term_bytes
    lens = np.diff(ix.term_off.astype(np.int64))
    assert (lens >= 1).all() and (lens <= 255).all(), "term length out of [1,255]"
    assert ix.post_off[0] == 0 and ix.post_off[-1] == ix.n_postings
    dfs = np.diff(ix.post_off.astype(np.int64))
    assert (dfs == ix.df.astype(np.int64)).all(), "df != post_off diff"
    assert (ix.df >= 1).all()
    assert int(ix.df.astype(np.int64).sum()) == ix.n_postings
    assert int(ix.cf.astype(np.uint64).sum()) == ix.n_tokens
    assert int(ix.tf.astype(np.uint64).sum()) == ix.n_tokens
    assert (ix.tf >= 1).all()
    if ix.n_postings:
        assert int(ix.docid.max()) < ix.n_docs
    # per-term tf sums equal cf and docIDs strictly increase within each list
    seg = np.repeat(np.arange(ix.n_terms), dfs)
    if ix.n_postings:
        sums = np.bincount(seg, weights=ix.tf.astype(np.float64), minlength=ix.n_terms)
        assert np.array_equal(sums.astype(np.uint64), ix.cf.astype(np.uint64)), "sum tf != cf"
        d = ix.docid.astype(np.int64)
        inc = np.diff(d) > 0
        same_term = np.diff(seg) == 0
        assert (inc | ~same_term).all(), "docIDs not strictly increasing within a list"
    terms = ix.terms()
    for a, b in zip(terms, terms[1:]):
        assert a < b, f"dictionary not strictly increasing: {a!r} >= {b!r}"
    for t in terms:
        assert all(not (65 <= c <= 90) for c in t), "unfolded upper-case byte"


def serialize(n_docs, n_tokens, n_dropped, terms, postings):
    """Canonical bytes from python lists (test helper): terms = [bytes], postings = [[(doc, tf)]]."""
    import struct

    out = bytearray(b"WJINV001")
    n_post = sum(len(p) for p in postings)
    tb = b"".join(terms)
    out += struct.pack("<7Q", n_docs, n_tokens, n_dropped, len(terms), n_post, len(tb), 0)
    off = 0
    for t in terms:
        out += struct.pack("<Q", off)
        off += len(t)
    out += struct.pack("<Q", off)
    out += tb + b"\0" * (_pad8(len(tb)) - len(tb))
    df = b"".join(struct.pack("<I", len(p)) for p in postings)
    out += df + b"\0" * (_pad8(len(df)) - len(df))
    for p in postings:
        out += struct.pack("<Q", sum(f for _, f in p))
    off = 0
    for p in postings:
        out += struct.pack("<Q", off)
        off += len(p)
    out += struct.pack("<Q", off)
    d = b"".join(struct.pack("<I", x) for p in postings for x, _ in p)
    out += d + b"\0" * (_pad8(len(d)) - len(d))
    f = b"".join(struct.pack("<I", y) for p in postings for _, y in p)
    out += f + b"\0" * (_pad8(len(f)) - len(f))
    return bytes(out)


def split_by_owner(buf: bytes, world: int, bucket_fn):
    """Slices of a serialized index: rank r keeps the terms of trie collections b with b % world == r."""
    ix = parse(buf)
    d = ix.as_dict()
    out = []
    for r in range(world):
        terms = [t for t in ix.terms() if bucket_fn(t) % world == r]
        posts = [d[t] for t in terms]
        ntok = sum(f for p in posts for _, f in p)
        out.append(serialize(ix.n_docs, ntok, ix.n_dropped if r == 0 else 0, terms, posts))
    return out
