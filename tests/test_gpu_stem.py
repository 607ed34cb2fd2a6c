"""Parser Steps 3-4 on the GPU (P:140 Porter stemmer, P:141 stop words; reading S20)
vs the CPU oracle, through the C ABI.

Bar: the device stemmer's output equals the oracle's Porter stem word for word; indexes built with
WJ_FLAG_STEM / WJ_FLAG_STOPWORDS are byte-identical to oracle.index_bytes(stem=, stop=) for every
chunking, on one GPU and through the multi-rank loopback path.
"""
import numpy as np
import pytest

import gen
import oracle
import wjformat
from golden_io import load_corpus

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_weij11_b200 as wj  # noqa: E402
from test_gpu_multi import dist_index  # noqa: E402
from test_gpu_parity import assert_same_index  # noqa: E402
from test_oracle import PORTER_STEP_EXAMPLES  # noqa: E402


def gpu_index(text, doc_off, cuts=None, **kw):
    off = np.asarray(doc_off, dtype=np.uint64)
    text = np.asarray(text, dtype=np.uint8)
    cuts = cuts or [0, len(off) - 1]
    with wj.Index(device=0, **kw) as ix:
        for a, b in zip(cuts, cuts[1:]):
            ix.add_stream(text[int(off[a]):int(off[b])], off[a:b + 1] - off[a])
        ix.finalize()
        return ix.serialize()


def test_device_porter_paper_examples():
    words = [w.encode() for step in PORTER_STEP_EXAMPLES.values() for w, _ in step]
    words += [b"generalizations", b"oscillators", b"is", b"as", b"3d", b"a\xc3\xb1os", b"abc1", b"y", b"yy",
              b"yyy", b"sky", b"syzygy", b"queueing", b"x" * 255, b"ies", b"sses", b"eed", b"ing", b"ed"]
    got = wj.debug_stem(words)
    assert got == [oracle.porter(w) for w in words]


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_device_porter_vs_oracle_many_words(seed):
    words = gen.suffix_rich_words(seed, 20000)
    words += [s.encode() for s in wj.stop_words()]
    assert wj.debug_stem(words) == [oracle.porter(w) for w in words]


def test_device_porter_generated_vocabulary():
    text, off = gen.generate(gen.CONFIGS[1])
    words = sorted({t for t in wjformat.parse(oracle.index_bytes(text, off)).terms()})
    assert wj.debug_stem(words) == [oracle.porter(w) for w in words]


@pytest.mark.parametrize("stem,stop", [(True, False), (False, True), (True, True)])
@pytest.mark.parametrize("name", ["corpus_survey.txt", "corpus_edges.txt"])
def test_golden_stem_stop(name, stem, stop):
    text, off = gen.from_docs(load_corpus(name)[0])
    assert_same_index(gpu_index(text, off, stem=stem, stop=stop), oracle.index_bytes(text, off, stem=stem, stop=stop))


@pytest.mark.parametrize("stem,stop", [(True, False), (False, True), (True, True)])
def test_suffix_rich_corpus(stem, stop):
    docs = gen.suffix_rich_docs(7, 600, stop_words=wj.stop_words())
    text, off = gen.from_docs(docs)
    want = oracle.index_bytes(text, off, stem=stem, stop=stop)
    assert_same_index(gpu_index(text, off, stem=stem, stop=stop), want)
    assert_same_index(gpu_index(text, off, cuts=[0, 1, 250, 251, 600], stem=stem, stop=stop), want)


def test_config1_stem_stop_multichunk():
    text, off = gen.generate(gen.CONFIGS[1])
    want = oracle.index_bytes(text, off, stem=True, stop=True)
    assert_same_index(gpu_index(text, off, cuts=[0, 333, 700, 1000], stem=True, stop=True), want)
    # stemming really changed the dictionary on this corpus
    assert want != oracle.index_bytes(text, off)


def test_all_stop_words_and_empty_chunks():
    docs = [b"The the THE a an", b"", b"of and to", b"cats", b"is IS is", b""]
    text, off = gen.from_docs(docs)
    for cuts in ([0, 6], [0, 1, 2, 3, 4, 5, 6], [0, 3, 6]):
        want = oracle.index_bytes(text, off, stem=True, stop=True)
        assert_same_index(gpu_index(text, off, cuts=cuts, stem=True, stop=True), want)
    text, off = gen.from_docs([b"the of and", b"a"])
    want = oracle.index_bytes(text, off, stop=True)
    got = gpu_index(text, off, stop=True)
    assert_same_index(got, want)
    assert wjformat.parse(got).n_tokens == 0


def test_read_postings_by_stem():
    docs = [b"Cats and dogs", b"a cat, the cats", b"generalizations"]
    text, off = gen.from_docs(docs)
    with wj.Index(device=0, stem=True, stop=True) as ix:
        ix.add_stream(text, off)
        ix.finalize()
        d, t = ix.read_postings(b"cat")
        assert d.tolist() == [0, 1] and t.tolist() == [1, 2]
        assert ix.read_postings(b"cats") is None
        assert ix.read_postings(b"and") is None
        assert ix.read_postings(b"gener")[0].tolist() == [2]


@pytest.mark.parametrize("K", [2, 3])
def test_loopback_stem_stop(K):
    docs = gen.suffix_rich_docs(11, 400, stop_words=wj.stop_words())
    text, off = gen.from_docs(docs)
    want = oracle.index_bytes(text, off, stem=True, stop=True)
    slices, _ = dist_index(text, off, K, cuts=[0, 150, 400], stem=True, stop=True)
    for r, sl in enumerate(slices):
        assert all(oracle.bucket(t) % K == r for t in wjformat.parse(sl).terms())
    assert wj.merge_serialized(slices) == want
