"""Multi-rank indexing through the C ABI on one GPU (loopback transport, one host thread per rank).

Each rank indexes its own contiguous document range of every chunk; terms are routed to the rank
owning their trie collection (b mod K) with the same pack / all-to-all-v / unpack code
the NCCL transport uses.  Parity: the merge of the K slices is byte-identical to the CPU oracle, and
every slice holds only owned collections.
"""
import threading

import numpy as np
import pytest

import gen
import oracle
import wjformat

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_weij11_b200 as wj  # noqa: E402


def dist_index(text, doc_off, K, cuts=None, queries=(), vbyte=False, balanced=False, maps=None, stem=False,
               stop=False, **kw):
    off = np.asarray(doc_off, dtype=np.uint64)
    text = np.asarray(text, dtype=np.uint8)
    n = len(off) - 1
    cuts = cuts or [0, n]
    hub = wj.LoopbackHub(K)
    slices = [None] * K
    answers = [dict() for _ in range(K)]
    errors = []

    def run(r):
        try:
            with wj.Index(device=0, rank=r, world=K, hub=hub, own_stream=True, vbyte=vbyte, balanced=balanced, stem=stem,
                          stop=stop, **kw) as ix:
                for a, b in zip(cuts, cuts[1:]):
                    # rank r's contiguous document range of this chunk (rank order = DocID order)
                    bounds = [a + (b - a) * i // K for i in range(K + 1)]
                    lo, hi = bounds[r], bounds[r + 1]
                    t = text[int(off[lo]):int(off[hi])]
                    o = off[lo:hi + 1] - off[lo]
                    ix.add_stream(t, o)
                ix.finalize()
                slices[r] = ix.serialize()
                if maps is not None:
                    maps[r] = ix.owner_map()
                for q in queries:
                    answers[r][q] = ix.read_postings(q)
        except Exception as e:  # pragma: no cover
            errors.append((r, e))
            raise

    th = [threading.Thread(target=run, args=(r,)) for r in range(K)]
    for x in th:
        x.start()
    for x in th:
        x.join(timeout=600)
    hub.close()
    assert not errors, errors
    return slices, answers


@pytest.mark.parametrize("K", [2, 3, 4, 8])
def test_loopback_config1(K):
    text, off = gen.generate(gen.CONFIGS[1])
    want = oracle.index_bytes(text, off)
    slices, _ = dist_index(text, off, K, cuts=[0, 400, 1000])
    for r, sl in enumerate(slices):
        ix = wjformat.parse(sl)
        assert all(oracle.bucket(t) % K == r for t in ix.terms()), "slice holds a non-owned collection"
        assert ix.n_docs == 1000
    assert wj.merge_serialized(slices) == want


@pytest.mark.parametrize("K", [1, 2, 3, 8])
@pytest.mark.parametrize("global_stream", [False, True])
def test_loopback_both_paths(K, global_stream):
    """Default: sender-side partial lists (every rank sorts its own stream by (owner, term) and sends
    per-term postings, P:160-162 / P:237); WJ_FLAG_GLOBAL_STREAM: token records routed to the owner and
    one global sort at finalize.  Both byte-identical to the oracle over three chunks."""
    text, off = gen.generate(gen.CONFIGS[1])
    want = oracle.index_bytes(text, off)
    slices, _ = dist_index(text, off, K, cuts=[0, 300, 301, 1000], global_stream=global_stream)
    assert wj.merge_serialized(slices) == want


@pytest.mark.parametrize("K", [2, 8])
def test_loopback_hot_terms(K):
    # opt-in hot-term merging on the senders (holes + count elements in the local sort)
    cfg = gen.CONFIGS[2].scaled(chunk_bytes=8 << 20, vocab=100_000)
    text, off = gen.generate(cfg)
    n = len(off) - 1
    slices, _ = dist_index(text, off, K, cuts=[0, n // 2, n], hot=True)
    assert wj.merge_serialized(slices) == oracle.index_bytes(text, off)


def test_loopback_k8_config3_shape_exchange_volume():
    """K = 8 on Wikipedia-shaped text (short documents): byte-identical merge, and the bytes sent
    stay below 8 B per token (postings aggregated per (term, document) plus term bytes and headers)."""
    cfg = gen.CONFIGS[3].scaled(chunk_bytes=16 << 20, vocab=200_000)
    text, off = gen.generate(cfg)
    n = len(off) - 1
    K = 8
    stats = [None] * K
    hub = wj.LoopbackHub(K)
    slices = [None] * K
    errors = []

    def run(r):
        try:
            with wj.Index(device=0, rank=r, world=K, hub=hub, own_stream=True) as ix:
                bounds = [n * i // K for i in range(K + 1)]
                lo, hi = bounds[r], bounds[r + 1]
                ix.add_stream(text[int(off[lo]):int(off[hi])], off[lo:hi + 1] - off[lo])
                ix.finalize()
                slices[r] = ix.serialize()
                stats[r] = ix.stats()
        except Exception as e:  # pragma: no cover
            errors.append((r, e))
            raise

    th = [threading.Thread(target=run, args=(r,)) for r in range(K)]
    for x in th:
        x.start()
    for x in th:
        x.join(timeout=600)
    hub.close()
    assert not errors, errors
    full = oracle.index_bytes(text, off)
    assert wj.merge_serialized(slices) == full
    sent = sum(s["exchange_bytes"] for s in stats)
    ntok = int(wjformat.parse(full).n_tokens)
    assert sent < 8 * ntok


def test_loopback_edges_and_queries():
    docs = [b"", b"a", b"b", b"Apple apple APPLE", b"x" * 300 + b" zoo 01 0195 954", b"", b"aaat aabomycin zzzy",
            b"application lication"] * 5
    text, off = gen.from_docs(docs)
    want = oracle.index_bytes(text, off)
    o = oracle.Oracle()
    o.add(text, off)
    qs = [b"apple", b"zoo", b"application", b"01", b"nothere"]
    slices, ans = dist_index(text, off, 3, cuts=[0, 7, 8, 40], queries=qs)
    assert wj.merge_serialized(slices) == want
    for q in qs:
        owner = oracle.bucket(q) % 3
        for r in range(3):
            got = ans[r][q]
            ref = o.postings(q)
            if r == owner and ref is not None:
                assert got is not None and np.array_equal(got[0], ref[0]) and np.array_equal(got[1], ref[1])
            else:
                assert got is None


def test_loopback_many_chunks_new_terms():
    cfg = gen.CONFIGS[1].scaled(vocab=80_000)
    text, off = gen.generate(cfg)
    want = oracle.index_bytes(text, off)
    slices, _ = dist_index(text, off, 2, cuts=[0, 3, 100, 101, 500, 1000])
    assert wj.merge_serialized(slices) == want


def test_loopback_rank_with_no_documents():
    text, off = gen.from_docs([b"one two three", b"two three four"])
    want = oracle.index_bytes(text, off)
    slices, _ = dist_index(text, off, 4)  # 2 documents over 4 ranks: two ranks send nothing
    assert wj.merge_serialized(slices) == want


def test_nccl_transport_single_rank():
    # world 1 with an NCCL communicator runs the distributed path (comm init, all-gather, self send/recv)
    text, off = gen.generate(gen.CONFIGS[1])
    want = oracle.index_bytes(text, off)
    nid = wj.nccl_unique_id()
    with wj.Index(device=0, rank=0, world=1, nccl_id=nid) as ix:
        ix.add_stream(text[: int(off[300])], off[:301])
        ix.add_stream(text[int(off[300]):], off[300:] - off[300])
        ix.finalize()
        got = ix.serialize()
        st = ix.stats()
    assert got == want
    assert st["exchange_bytes"] == 0  # nothing leaves a single rank


def test_loopback_single_rank():
    text, off = gen.generate(gen.CONFIGS[1].scaled(vocab=3000))
    slices, _ = dist_index(text, off, 1, cuts=[0, 500, 1000])
    assert slices[0] == oracle.index_bytes(text, off)


@pytest.mark.parametrize("K", [2, 3])
def test_loopback_vbyte_merge(K):
    # compressed slices (WJINV002) merge by concatenating each list's self-contained code
    text, off = gen.generate(gen.CONFIGS[1])
    slices, _ = dist_index(text, off, K, cuts=[0, 500, 1000], vbyte=True)
    assert wj.merge_serialized(slices) == oracle.index_bytes(text, off, vbyte=True)


def test_loopback_host_pipeline():
    # every rank defers its host chunks by one call; collectives still pair up in chunk order
    text, off = gen.generate(gen.CONFIGS[1])
    off = np.asarray(off, dtype=np.uint64)
    K = 2
    hub = wj.LoopbackHub(K)
    slices = [None] * K
    errors = []

    def run(r):
        try:
            with wj.Index(device=0, rank=r, world=K, hub=hub, own_stream=True, pipeline=True) as ix:
                for a, b in zip([0, 300, 700], [300, 700, 1000]):
                    bounds = [a + (b - a) * i // K for i in range(K + 1)]
                    lo, hi = bounds[r], bounds[r + 1]
                    ix.add_stream(text[int(off[lo]):int(off[hi])].copy(), off[lo:hi + 1] - off[lo])
                ix.finalize()
                slices[r] = ix.serialize()
        except Exception as e:  # pragma: no cover
            errors.append((r, e))
            raise

    th = [threading.Thread(target=run, args=(r,)) for r in range(K)]
    for x in th:
        x.start()
    for x in th:
        x.join(timeout=600)
    hub.close()
    assert not errors, errors
    assert wj.merge_serialized(slices) == oracle.index_bytes(text, off)


@pytest.mark.parametrize("K", [3, 4, 8])
def test_loopback_balanced_owner_map(K):
    # sampled bin-packing of the trie collections: same map on every rank, every slice
    # holds exactly its collections, the merge is the oracle's file, and the sampled-token load of
    # the busiest rank is close to the mean
    cfg = gen.CONFIGS[2].scaled(chunk_bytes=12 << 20, vocab=300_000)
    text, off = gen.generate(cfg)
    n = len(off) - 1
    maps = [None] * K
    slices, _ = dist_index(text, off, K, cuts=[0, n // 2, n], balanced=True, maps=maps)
    assert all(np.array_equal(maps[0], m) for m in maps)
    assert not np.array_equal(maps[0], np.arange(wj.N_COLLECTIONS) % K)
    for r, sl in enumerate(slices):
        ix = wjformat.parse(sl)
        assert all(maps[0][oracle.bucket(t)] == r for t in ix.terms())
    assert wj.merge_serialized(slices) == oracle.index_bytes(text, off)
    load = np.array([int(wjformat.parse(sl).n_tokens) for sl in slices], dtype=np.float64)
    mod = np.zeros(K)
    full = wjformat.parse(oracle.index_bytes(text, off))
    for t, c in zip(full.terms(), full.cf):
        mod[oracle.bucket(t) % K] += int(c)
    assert load.max() / load.mean() < 1.10
    assert load.max() / load.mean() <= mod.max() / mod.mean() + 1e-9
