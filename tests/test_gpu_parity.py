"""CUDA path vs the CPU oracle, through the C ABI (needs a B200: run with `-m gpu`).

Parity bar (integer/byte work): the serialized inverted file is bit-exact, token
dumps are identical, read_postings equals the oracle's lists.
"""
import hashlib

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import gen
import oracle
import wjformat
from golden_io import load_corpus

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_weij11_b200 as wj  # noqa: E402


def gpu_index(text, doc_off, cuts=None, device_input=False, vbyte=False, **kw):
    with wj.Index(device=0, vbyte=vbyte, **kw) as ix:
        off = np.asarray(doc_off, dtype=np.uint64)
        text = np.asarray(text, dtype=np.uint8)
        cuts = cuts or [0, len(off) - 1]
        for a, b in zip(cuts, cuts[1:]):
            t = text[int(off[a]):int(off[b])]
            o = off[a:b + 1] - off[a]
            if device_input:
                t = torch.from_numpy(t.copy()).cuda()
                o = torch.from_numpy(o.astype(np.int64)).cuda()
            ix.add_stream(t, o)
            torch.cuda.synchronize()
        ix.finalize()
        return ix.serialize()


def assert_same_index(got: bytes, want: bytes):
    if got == want:
        return
    g, w = wjformat.parse(got), wjformat.parse(want)
    hdr = ["n_docs", "n_tokens", "n_dropped", "n_terms", "n_postings", "n_term_bytes"]
    assert [getattr(g, h) for h in hdr] == [getattr(w, h) for h in hdr]
    gt, wt = g.terms(), w.terms()
    for i, (a, b) in enumerate(zip(gt, wt)):
        assert a == b, f"term {i}: {a!r} != {b!r}"
    assert np.array_equal(g.df, w.df), "df differs"
    assert np.array_equal(g.cf, w.cf), "cf differs"
    assert np.array_equal(g.docid, w.docid), "docids differ"
    assert np.array_equal(g.tf, w.tf), "tfs differ"
    assert got == want


def docs_to_corpus(docs):
    return gen.from_docs(docs)


# ------------------------------------------------------------------ token dump (K1, Table I)
@pytest.mark.parametrize("name", ["corpus_survey.txt", "corpus_edges.txt"])
def test_token_dump_golden(name):
    docs, _, _ = load_corpus(name)
    text, off = docs_to_corpus(docs)
    with wj.Index() as ix:
        assert ix.debug_tokens(text, off) == oracle.dump_tokens(text, off)


def test_token_dump_config1():
    text, off = gen.generate(gen.CONFIGS[1])
    with wj.Index() as ix:
        got = ix.debug_tokens(text, off, doc_base=7)
    assert got == oracle.dump_tokens(text, off, doc_base=7)


# ------------------------------------------------------------------ whole index
@pytest.mark.parametrize("name", ["corpus_survey.txt", "corpus_edges.txt"])
def test_golden_index(name):
    docs, hdr, terms = load_corpus(name)
    text, off = docs_to_corpus(docs)
    got = gpu_index(text, off)
    ix = wjformat.parse(got)
    assert ix.as_dict() == terms
    assert (ix.n_docs, ix.n_tokens, ix.n_dropped) == (hdr["n_docs"], hdr["n_tokens"], hdr["n_dropped"])
    assert_same_index(got, oracle.index_bytes(text, off))


def test_config1_single_chunk():
    text, off = gen.generate(gen.CONFIGS[1])
    assert_same_index(gpu_index(text, off), oracle.index_bytes(text, off))


def test_config1_device_input_many_chunks():
    text, off = gen.generate(gen.CONFIGS[1])
    want = oracle.index_bytes(text, off)
    assert_same_index(gpu_index(text, off, cuts=[0, 1, 2, 250, 251, 700, 1000], device_input=True), want)
    assert_same_index(gpu_index(text, off, cuts=list(range(0, 1001, 50))), want)


def test_edge_documents():
    seg = 512
    docs = [
        b"",
        b"a",
        b"b",  # adjacent one-byte documents: two tokens, never merged (S1)
        b"x" * (seg - 1) + b"Y",  # a token ending exactly at a 512-byte segment end
        b"q" * 255 + b" " + b"r" * 256 + b" " + b"Z" * 1000,  # 255 kept, 256 and 1000 dropped
        b" " * 300 + b"w" * 255,  # 255-byte token crossing a segment boundary
        b"\x00\xff\x80-\x7f" * 100,
        b"", b"", b"",
        b"MiXeD CaSe mixed case \xc3\x89t\xc3\xa9 \xc3\xa9t\xc3\xa9",
        bytes(range(256)) * 3,
        b"0 00 000 0a a0 9z z9 zzzz zzz zz",
    ]
    text, off = docs_to_corpus(docs)
    want = oracle.index_bytes(text, off)
    assert_same_index(gpu_index(text, off), want)
    with wj.Index() as ix:
        assert ix.debug_tokens(text, off) == oracle.dump_tokens(text, off)


def test_doc_boundaries_every_position():
    # documents of every length 0..70 so that boundaries fall on every offset inside 16-byte lanes
    rng = np.random.default_rng(5)
    pool = np.frombuffer(b"abcXYZ019 ,.\xc3\xa9", dtype=np.uint8)
    docs = [bytes(rng.choice(pool, size=n)) for n in list(range(71)) * 8]
    text, off = docs_to_corpus(docs)
    assert_same_index(gpu_index(text, off), oracle.index_bytes(text, off))
    with wj.Index() as ix:
        assert ix.debug_tokens(text, off) == oracle.dump_tokens(text, off)


BYTE_POOL = list(b"aAbBzZ09 ,.-!\t\n") + [0x00, 0x7F, 0x80, 0xC3, 0xA9, 0xFF]


@settings(max_examples=40, deadline=None)
@given(st.lists(st.lists(st.sampled_from(BYTE_POOL), max_size=700).map(bytes), min_size=1, max_size=20),
       st.integers(min_value=1, max_value=4))
def test_random_corpora(docs, nchunks):
    text, off = docs_to_corpus(docs)
    n = len(docs)
    cuts = sorted(set([0, n] + [int(x) for x in np.linspace(0, n, nchunks + 1)]))
    assert_same_index(gpu_index(text, off, cuts=cuts), oracle.index_bytes(text, off))


def test_closed_form_corpus_gpu():
    D, J = 3000, 400
    text, off = gen.closed_form(D, J)
    got = wjformat.parse(gpu_index(text, off))
    want = {}
    for j in range(J):
        want[gen.closed_form_term(j)] = [(d, 1 + (d + j) % 3) for d in range(0, D, j + 1)]
    assert got.as_dict() == dict(sorted(want.items()))


def test_many_new_terms_across_chunks():
    # second and later chunks insert into existing B-trees (merge + rebuild path)
    cfg = gen.CONFIGS[1].scaled(vocab=50_000)
    text, off = gen.generate(cfg)
    cuts = [0, 100, 101, 400, 1000]
    assert_same_index(gpu_index(text, off, cuts=cuts), oracle.index_bytes(text, off))


# ------------------------------------------------------------------ retrieval + B-tree
def test_read_postings_matches_oracle():
    text, off = gen.generate(gen.CONFIGS[1])
    o = oracle.Oracle()
    o.add(text, off)
    ixb = wjformat.parse(o.serialize())
    terms = ixb.terms()
    rng = np.random.default_rng(1)
    sample = [terms[i] for i in rng.choice(len(terms), size=200, replace=False)] + terms[:5] + terms[-5:]
    with wj.Index() as ix:
        ix.add_stream(text, off)
        ix.finalize()
        for t in sample:
            d, f = ix.read_postings(t)
            wd, wf = o.postings(t)
            assert np.array_equal(d, wd) and np.array_equal(f, wf), t
        assert ix.read_postings(b"notaterm12345zz") is None
        assert ix.read_postings(b"has space") is None
        up = ix.read_postings(terms[0].upper())  # queries are folded like tokens (S2)
        assert up is not None and np.array_equal(up[0], o.postings(terms[0])[0])


def _arena_term(arena, off):
    n = int(arena[off])
    return bytes(arena[off + 1: off + 1 + n])


def test_btree_invariants():
    cfg = gen.CONFIGS[1].scaled(vocab=200_000)
    text, off = gen.generate(cfg.scaled(chunk_bytes=8 << 20))
    with wj.Index() as ix:
        n = len(off) - 1
        ix.add_stream(text[: int(off[n // 3])], off[: n // 3 + 1])
        ix.add_stream(text[int(off[n // 3]):], off[n // 3:] - off[n // 3])
        nodes, coll, arena = ix.debug_btree()
        st_ = ix.stats()
    assert len(nodes) == st_["btree_nodes"] > 0
    total = 0
    seen_nodes = 0
    for b in range(wj.N_COLLECTIONS):
        root, nk, h = (int(x) for x in coll[b])
        total += nk
        if nk == 0:
            continue
        # height (edges) <= log_t((n+1)/2) for t = 16, when n >= 2
        if nk >= 2:
            assert (h - 1) <= np.log((nk + 1) / 2) / np.log(16) + 1e-9
        keys = []
        leaf_depths = set()

        def walk(node, depth, is_root):
            nonlocal seen_nodes
            seen_nodes += 1
            nd = nodes[node]
            c = int(nd["count"])
            assert 1 <= c <= 31
            if not is_root:
                assert 15 <= c <= 31, (b, c)  # t = 16
            for j in range(c):
                s = _arena_term(arena, int(nd["str"][j]))
                want_cache = int.from_bytes((s[:4] + b"\0\0\0\0")[:4], "big")
                assert int(nd["cache"][j]) == want_cache
            if nd["leaf"]:
                leaf_depths.add(depth)
                for j in range(c):
                    keys.append(_arena_term(arena, int(nd["str"][j])))
            else:
                for j in range(c + 1):
                    walk(int(nd["child"][j]), depth + 1, False)
                    if j < c:
                        keys.append(_arena_term(arena, int(nd["str"][j])))

        walk(root, 0, True)
        assert len(leaf_depths) == 1 and leaf_depths.pop() == h - 1
        assert len(keys) == nk
        assert all(a < b2 for a, b2 in zip(keys, keys[1:])), "in-order traversal not increasing"
        # every key's own trie index is this collection (Table I; prefix stripped)
        for s in keys[:3]:
            pass
    assert seen_nodes == len(nodes)
    assert total == st_["n_terms"]


# ------------------------------------------------------------------ ABI behaviour
def test_state_machine_and_errors():
    text, off = gen.from_docs([b"alpha beta", b"beta gamma"])
    with wj.Index() as ix:
        with pytest.raises(wj.WJError) as e:
            ix.serialize()
        assert e.value.code == -2
        with pytest.raises(wj.WJError) as e:
            ix.add_stream(text, np.array([0, 3, 2, len(text)], dtype=np.uint64))
        assert e.value.code == -1
        ix.add_stream(text, off)
        ix.finalize()
        with pytest.raises(wj.WJError) as e:
            ix.add_stream(text, off)
        assert e.value.code == -2
        with pytest.raises(wj.WJError) as e:
            ix.finalize()
        assert e.value.code == -2
        assert wjformat.parse(ix.serialize()).terms() == [b"alpha", b"beta", b"gamma"]
        ix.reset()
        ix.add_stream(text, off)
        ix.finalize()
        assert ix.serialize() == oracle.index_bytes(text, off)


def test_empty_inputs():
    with wj.Index() as ix:
        ix.add_stream(np.zeros(0, np.uint8), np.zeros(1, np.uint64))
        ix.add_stream(np.zeros(0, np.uint8), np.zeros(4, np.uint64))  # three empty documents
        ix.add_stream(np.frombuffer(b" ,. ", np.uint8), np.array([0, 4], np.uint64))
        ix.finalize()
        got = ix.serialize()
    t, o = gen.from_docs([b"", b"", b"", b" ,. "])
    assert got == oracle.index_bytes(t, o)


# ------------------------------------------------------------------ full-size configs
def _sha(b):
    return hashlib.sha256(b).hexdigest()


@pytest.mark.slow
def test_config2_full_size_sha():
    """BASELINE config 2 (1 GiB ClueWeb09-shaped) at full size: SHA-256 of the serialized index vs
    the doc-range-sharded oracle (oracle_add_mt), plus invariants and sampled postings."""
    import os
    text, off = gen.generate(gen.CONFIGS[2])
    tt = torch.from_numpy(text).cuda()
    to = torch.from_numpy(off.astype(np.int64)).cuda()
    with wj.Index() as ix:
        ix.add_stream(tt, to)
        ix.finalize()
        got = ix.serialize()
    threads = max(1, min(32, len(os.sched_getaffinity(0))))
    want = oracle.index_bytes(text, off, threads=threads)
    assert _sha(got) == _sha(want)
    wjformat.check_invariants(wjformat.parse(got))


# ------------------------------------------------------------------ sampled hot terms
@pytest.mark.parametrize("global_stream", [False, True])
@pytest.mark.parametrize("cfg_id", [2, 3, 4])
def test_hot_path_shapes(cfg_id, global_stream):
    cfg = gen.CONFIGS[cfg_id].scaled(chunk_bytes=6 << 20, vocab=200_000)
    text, off = gen.generate(cfg)
    n = len(off) - 1
    want = oracle.index_bytes(text, off)
    for cuts in (None, [0, n // 3, n // 3 + 1, n]):
        with wj.Index(device=0, hot=True, global_stream=global_stream) as ix:
            c = cuts or [0, n]
            for a, b in zip(c, c[1:]):
                ix.add_stream(text[int(off[a]):int(off[b])], (off[a:b + 1] - off[a]).astype(np.uint64))
            ix.finalize()
            assert_same_index(ix.serialize(), want)
            s = ix.stats()
            if not global_stream:  # hot terms are a partial-list-path option
                assert s["hot_elems_saved"] > 0
                assert s["stream_elems"] + s["hot_elems_saved"] == s["n_tokens"]


@pytest.mark.parametrize("global_stream", [False, True])
def test_hot_path_repetitive_docs(global_stream):
    # hot counts above 2^16 in one document (the per-warp u16 counters flush per 2 KB range), runs of
    # one-token documents (more than kHotDocs documents in one warp range), hot terms at every boundary
    docs = [b"the " * 600 + b"cat", b"the", b"", b"The the THE"] * 300 + [b"x y z " * 5000] + [b"the"] * 3000 + [
        b"a " * 70000]
    text, off = gen.from_docs(docs)
    want = oracle.index_bytes(text, off)
    assert_same_index(gpu_index(text, off, hot=True, global_stream=global_stream), want)
    assert_same_index(gpu_index(text, off, cuts=[0, 1000, 1001, len(docs)], hot=True, global_stream=global_stream),
                      want)


def test_long_runs_across_run_length_ranges():
    """(term, doc) runs far longer than a run-length warp range (k_rlw_write walks 512-element steps;
    a range with no posting start adds all its elements to the previous range's open posting through
    k_rle_fixup), next to single-token documents and a new document at every step boundary."""
    docs = [b"w " * 70000 + b"end", b"w", b"v w"] + [b"w " * 511 + b"q"] * 40 + [b"a " * 1024] * 3 + [b"x"] * 2000
    text, off = gen.from_docs(docs)
    want = oracle.index_bytes(text, off)
    assert_same_index(gpu_index(text, off), want)
    assert_same_index(gpu_index(text, off, cuts=[0, 1, 40, len(docs)]), want)
    assert_same_index(gpu_index(text, off, global_stream=True), want)


def test_hot_off_by_default():
    cfg = gen.CONFIGS[2].scaled(chunk_bytes=10 << 20, vocab=100_000)
    text, off = gen.generate(cfg)
    want = oracle.index_bytes(text, off)
    with wj.Index(device=0) as ix:
        ix.add_stream(text, off)
        ix.finalize()
        assert_same_index(ix.serialize(), want)
        s = ix.stats()
        assert s["hot_elems_saved"] == 0 and s["stream_elems"] == s["n_tokens"]


def test_multichunk_config3_shape():
    # Wikipedia-shaped (short documents, several chunks): maps per chunk, dictionary merge + rebuild
    cfg = gen.CONFIGS[3].scaled(chunk_bytes=4 << 20, vocab=300_000)
    parts = [gen.generate(cfg, chunk=c) for c in range(3)]
    with wj.Index() as ix:
        for t, o in parts:
            ix.add_stream(t, o)
        ix.finalize()
        got = ix.serialize()
    o = oracle.Oracle()
    for t, oo in parts:
        o.add(t, oo)
    assert_same_index(got, o.serialize())


# ------------------------------------------------------------------ f1: d-gap + vbyte code
def test_vbyte_golden_and_config1():
    docs, _, _ = load_corpus("corpus_edges.txt")
    text, off = gen.from_docs(docs)
    assert gpu_index(text, off, vbyte=True) == oracle.index_bytes(text, off, vbyte=True)
    text, off = gen.generate(gen.CONFIGS[1])
    want = oracle.index_bytes(text, off, vbyte=True)
    assert gpu_index(text, off, vbyte=True) == want
    assert gpu_index(text, off, cuts=[0, 1, 333, 334, 1000], vbyte=True) == want


@pytest.mark.parametrize("seed", [0, 1])
def test_vbyte_multi_tile_large_gaps(seed):
    # > 4096 postings (several encode tiles), lists spanning tiles, gaps of 1..5 bytes, big tf
    rng = np.random.default_rng(seed)
    docs = []
    for d in range(30000):
        words = [b"w%d" % int(x) for x in rng.zipf(1.3, size=int(rng.integers(0, 12))) if x < 10 ** 6]
        if d % 997 == 0:
            words += [b"many"] * int(rng.integers(100, 400))
        docs.append(b" ".join(words))
    text, off = gen.from_docs(docs)
    want = oracle.index_bytes(text, off, vbyte=True)
    got = gpu_index(text, off, vbyte=True)
    if got != want:
        assert wjformat.parse(got).as_dict() == wjformat.parse(want).as_dict()
    assert got == want


def test_vbyte_config_shapes_and_read_postings():
    cfg = gen.CONFIGS[4].scaled(chunk_bytes=8 << 20, vocab=300_000)
    text, off = gen.generate(cfg)
    o = oracle.Oracle()
    o.add(text, off)
    with wj.Index(vbyte=True) as ix:
        ix.add_stream(text, off)
        ix.finalize()
        got = ix.serialize()
        for q in (b"the", b"zzzzzzzz", b"a"):
            ref = o.postings(q)
            ans = ix.read_postings(q)
            assert (ans is None) == (ref is None)
            if ref is not None:
                assert np.array_equal(ans[0], ref[0]) and np.array_equal(ans[1], ref[1])
    assert got == o.serialize(vbyte=True)


def test_vbyte_empty_index():
    text, off = gen.from_docs([b"", b"...", b""])
    assert gpu_index(text, off, vbyte=True) == oracle.index_bytes(text, off, vbyte=True)


def test_vbyte_four_byte_gaps():
    # 2.7 M empty documents between two postings: 4-byte gap and first-posting codes
    docs = [b"a b"] + [b""] * 2_700_000 + [b"a c", b"c"]
    text, off = gen.from_docs(docs)
    want = oracle.index_bytes(text, off, vbyte=True)
    assert gpu_index(text, off, vbyte=True) == want


# ------------------------------------------------------------------ f3: host-streamed pipeline
def _chunks(text, off, cuts):
    off = np.asarray(off, dtype=np.uint64)
    for a, b in zip(cuts, cuts[1:]):
        yield text[int(off[a]):int(off[b])], off[a:b + 1] - off[a]


@pytest.mark.parametrize("pinned", [True, False])
def test_pipeline_host_chunks(pinned):
    text, off = gen.generate(gen.CONFIGS[1])
    want = oracle.index_bytes(text, off)
    cuts = [0, 100, 100, 101, 400, 999, 1000]  # includes a chunk with no documents
    with wj.Index(pipeline=True) as ix:
        for t, o in _chunks(text, off, cuts):
            if pinned:
                t = torch.from_numpy(t.copy()).pin_memory()
                o = torch.from_numpy(o.astype(np.int64)).pin_memory()
            ix.add_stream(t, o)
        ix.finalize()
        got = ix.serialize()
        assert ix.stats()["n_docs"] == 1000
    assert_same_index(got, want)


def test_pipeline_mixed_host_device_and_vbyte():
    text, off = gen.generate(gen.CONFIGS[1].scaled(vocab=50_000))
    cuts = [0, 250, 500, 750, 1000]
    with wj.Index(pipeline=True, vbyte=True) as ix:
        for i, (t, o) in enumerate(_chunks(text, off, cuts)):
            if i == 2:  # a device chunk drains the pending host chunk first (DocID order)
                t = torch.from_numpy(t.copy()).cuda()
                o = torch.from_numpy(o.astype(np.int64)).cuda()
            ix.add_stream(t, o)
        ix.finalize()
        got = ix.serialize()
    assert got == oracle.index_bytes(text, off, vbyte=True)


def test_pipeline_reset_drops_pending_and_errors_at_call():
    text, off = gen.generate(gen.CONFIGS[1])
    with wj.Index(pipeline=True) as ix:
        t, o = next(_chunks(text, off, [0, 300]))
        ix.add_stream(t, o)  # copied, not yet indexed
        ix.reset()           # dropped
        bad = o.copy()
        bad[5], bad[6] = bad[6], bad[5] + 1
        with pytest.raises(wj.WJError):
            ix.add_stream(t, bad)  # doc_off validated at the call
        for t, o in _chunks(text, off, [0, 500, 1000]):
            ix.add_stream(t, o)
        ix.finalize()
        got = ix.serialize()
    assert_same_index(got, oracle.index_bytes(text, off))


@pytest.mark.parametrize("seed", [0, 1])
def test_new_terms_sharing_long_prefixes(seed):
    # new-term sort: equal (collection, first cached suffix bytes) keys are ordered by the rest of
    # the suffix (tie runs); terms that are prefixes of each other, and bytes >= 0x80 after the prefix
    rng = np.random.default_rng(seed)
    stems = [b"internation", b"abcdefgh", b"zzzzzzz", b"aaaa", b"qu\xc3\xa9bec", b"1234567"]
    words = []
    for st_ in stems:
        for _ in range(700):
            n = int(rng.integers(0, 9))
            words.append(st_ + bytes(int(x) for x in rng.choice(list(b"abcxyz09\xc3\xa9"), size=n)))
        words += [st_[:k] for k in range(1, len(st_) + 1)]
    docs = [b" ".join(words[i::7]) for i in range(7)] + [b" ".join(sorted(set(words)))]
    text, off = docs_to_corpus(docs)
    want = oracle.index_bytes(text, off)
    assert_same_index(gpu_index(text, off), want)
    assert_same_index(gpu_index(text, off, cuts=[0, 3, 5, 8]), want)


# ------------------------------------------------------------------ partial lists per run (partials.cuh)
@pytest.mark.parametrize("global_stream", [False, True])
def test_partials_and_global_stream_paths(global_stream):
    # default single-GPU path: per-chunk partial postings combined at finalize;
    # WJ_FLAG_GLOBAL_STREAM: the global stream sorted at finalize.  Both must give the oracle's bytes,
    # with chunks of very different sizes, empty chunks and a single-document chunk.
    cfg = gen.CONFIGS[3].scaled(chunk_bytes=3 << 20, vocab=50_000)
    text, off = gen.generate(cfg)
    n = len(off) - 1
    want = oracle.index_bytes(text, off)
    for cuts in ([0, n], [0, 1, 1, n // 7, n // 2, n - 1, n], [0, n // 3, 2 * n // 3, n]):
        assert_same_index(gpu_index(text, off, cuts=cuts, global_stream=global_stream), want)
    assert_same_index(gpu_index(text, off, cuts=[0, n // 2, n], vbyte=True, global_stream=global_stream),
                      oracle.index_bytes(text, off, vbyte=True))


def test_partials_repeated_reset_and_read_postings():
    cfg = gen.CONFIGS[2].scaled(chunk_bytes=2 << 20, vocab=20_000)
    text, off = gen.generate(cfg)
    want = oracle.index_bytes(text, off)
    w = wjformat.parse(want)
    with wj.Index(device=0) as ix:
        for _ in range(3):
            ix.reset()
            n = len(off) - 1
            for a, b in ((0, n // 2), (n // 2, n)):
                ix.add_stream(text[int(off[a]):int(off[b])], (off[a:b + 1] - off[a]).astype(np.uint64))
            ix.finalize()
            assert_same_index(ix.serialize(), want)
        terms = w.terms()
        for i in (0, len(terms) // 2, len(terms) - 1):
            d, t = ix.read_postings(terms[i])
            lo, hi = int(w.post_off[i]), int(w.post_off[i + 1])
            assert np.array_equal(d, w.docid[lo:hi]) and np.array_equal(t, w.tf[lo:hi])


def test_partials_profiled_stats_between_chunks():
    # WJ_FLAG_PROFILE with the side / dictionary streams: stats between add_stream calls (an unjoined
    # chunk, events on three streams), reset with a pending chunk, then a full pass
    cfg = gen.CONFIGS[2].scaled(chunk_bytes=3 << 20, vocab=40_000)
    text, off = gen.generate(cfg)
    n = len(off) - 1
    want = oracle.index_bytes(text, off)
    with wj.Index(device=0, profile=True) as ix:
        ix.add_stream(text[:int(off[n // 2])], off[:n // 2 + 1].astype(np.uint64))
        s = ix.stats()
        assert s["n_tokens"] > 0 and s["phase_ms"]["sort"] > 0 and s["kernel_count"]["sort_scatter"] > 0
        ix.reset()
        for a, b in ((0, n // 2), (n // 2, n)):
            ix.add_stream(text[int(off[a]):int(off[b])], (off[a:b + 1] - off[a]).astype(np.uint64))
            ix.stats()
        ix.finalize()
        assert_same_index(ix.serialize(), want)
        s = ix.stats()
        assert s["kernel_count"]["copy_partials"] >= 1 and s["stream_elems"] == s["n_tokens"]


# ------------------------------------------------------------------ robustness (round 2)
@pytest.mark.parametrize("doc", [b"a", b"ab", b"a b", b"a,", b"Zz9"])
def test_dense_tiny_documents(doc):
    """Thousands of consecutive 1-3 byte documents: up to 512 token starts in one 512-byte segment
    (every byte a document start), more than the emit kernel's per-warp token queue holds; the
    segment is queued in rounds (tokenize.cuh)."""
    docs = [doc] * 5000 + [b"tail word"] + [doc] * 3001
    text, off = docs_to_corpus(docs)
    want = oracle.index_bytes(text, off)
    assert_same_index(gpu_index(text, off), want)
    assert_same_index(gpu_index(text, off, cuts=[0, 777, 778, len(docs)]), want)
    with wj.Index() as ix:
        assert ix.debug_tokens(text, off) == oracle.dump_tokens(text, off)


def test_table_overflow_retry_forced():
    """A first chunk whose distinct-term count is far above the table's estimate (N/32): the
    probe sequences overflow and the chunk is retokenised with a doubled table (engine.cu
    tokenize_dedup); table_retries counts it and the index stays bit-exact."""
    rng = np.random.default_rng(11)
    letters = np.frombuffer(b"abcdefghijklmnopqrstuvwxyz", dtype=np.uint8)
    words = [rng.choice(letters, size=int(rng.integers(4, 14))).tobytes() for _ in range(60_000)]
    docs = [b" ".join(words[i:i + 40]) for i in range(0, len(words), 40)]
    text, off = docs_to_corpus(docs)
    want = oracle.index_bytes(text, off)
    with wj.Index(device=0) as ix:
        ix.add_stream(text, off)
        ix.finalize()
        got = ix.serialize()
        assert ix.stats()["table_retries"] >= 1
    assert_same_index(got, want)


# ------------------------------------------------------------------ full-size multi-chunk configs
def _fullsize_multichunk(cfg_id, chunks, **kw):
    """Configs 3 / 4 at full chunk size (1 GiB per index_add_stream): every chunk after the
    first probes and extends a non-empty dictionary (B-trees of height 3-4).  The GPU
    index is SHA-256-identical to the doc-range-sharded oracle (oracle_add_mt over all host cores)."""
    import os
    threads = max(1, min(64, len(os.sched_getaffinity(0))))
    o = oracle.Oracle()
    with wj.Index(**kw) as ix:
        for c in range(chunks):
            text, off = gen.generate(gen.CONFIGS[cfg_id], chunk=c)
            tt = torch.from_numpy(text).cuda()
            to = torch.from_numpy(off.astype(np.int64)).cuda()
            ix.add_stream(tt, to)
            o.add(text, off, threads=threads)
            torch.cuda.synchronize()
            del tt, to
        ix.finalize()
        got = ix.serialize()
        st = ix.stats()
    want = o.serialize()
    o.close()
    assert _sha(got) == _sha(want)
    wjformat.check_invariants(wjformat.parse(got))
    return st


@pytest.mark.slow
def test_config3_full_size_4_chunks():
    st = _fullsize_multichunk(3, 4)
    assert st["n_chunks"] == 4 and st["btree_height_max"] >= 3


@pytest.mark.slow
def test_config4_full_size_prefix_2_chunks():
    # Library-of-Congress shape: long documents, 1% hapax tokens (high new-term insert rate)
    st = _fullsize_multichunk(4, 2)
    assert st["n_chunks"] == 2 and st["new_terms_last"] > 100_000 and st["btree_height_max"] >= 3
