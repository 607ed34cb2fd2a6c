"""Pins for the CPU oracle against things other than itself (CPU only, `-m "not gpu"`).

Each test names what fixes the expected value: the paper's worked examples (Table I, the
"application" example), hand-counted corpora (tests/golden/), library routines (Python `re`
tokenisation + Counter brute force, coreutils tr|sort|uniq), a closed-form corpus and the
invariants of SURVEY.md §8(c).
"""
import re
import shutil
import subprocess
from collections import Counter, defaultdict

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import gen
import oracle
import wjformat
from golden_io import load_buckets, load_corpus

TOKEN_RE = re.compile(rb"[0-9A-Za-z\x80-\xff]+")


def brute_force(docs):
    """Independent definition: `re` tokenisation + bytes.lower() (ASCII-only) + counting."""
    post = defaultdict(list)
    n_tokens = n_dropped = 0
    for d, doc in enumerate(docs):
        cnt = Counter()
        for m in TOKEN_RE.findall(doc):
            if len(m) > 255:
                n_dropped += 1
                continue
            cnt[m.lower()] += 1
            n_tokens += 1
        for t, c in cnt.items():
            post[t].append((d, c))
    return {t: sorted(v) for t, v in post.items()}, n_tokens, n_dropped


def oracle_index(docs, threads=1):
    text, off = gen.from_docs(docs)
    ix = wjformat.parse(oracle.index_bytes(text, off, threads))
    wjformat.check_invariants(ix)
    return ix


# ---------------------------------------------------------------- Table I
@pytest.mark.parametrize("term,expected,cite", load_buckets())
def test_table1_examples(term, expected, cite):
    assert oracle.bucket(term) == expected, cite


def test_table1_printed_garble_is_not_row_11():
    # P:97 prints "afonuevo" under index 11; under the table's own rule it is 'afo' -> 181.
    # Reading S6: extraction garble of "añonuevo".  Pin the rule, not the garble.
    assert oracle.bucket(b"afonuevo") == 37 + 0 * 676 + 5 * 26 + 14


def test_table1_collection_count():
    # 1 special + 10 pure-number + 26 short/special + 26^3 = 17,613 collections (Table I).
    seen = {oracle.bucket(b"-")}
    seen |= {oracle.bucket(bytes([d])) for d in range(ord("0"), ord("9") + 1)}
    letters = range(ord("a"), ord("z") + 1)
    seen |= {oracle.bucket(bytes([a])) for a in letters}
    seen |= {oracle.bucket(bytes([a, b, c, ord("e")])) for a in letters for b in letters for c in letters}
    assert len(seen) == 17613 and min(seen) == 0 and max(seen) == 17612


# ---------------------------------------------------------------- hand-counted corpora
@pytest.mark.parametrize("name", ["corpus_survey.txt", "corpus_edges.txt"])
def test_hand_counted(name):
    docs, hdr, terms = load_corpus(name)
    ix = oracle_index(docs)
    assert ix.n_docs == hdr["n_docs"]
    assert ix.n_tokens == hdr["n_tokens"]
    assert ix.n_dropped == hdr["n_dropped"]
    assert ix.as_dict() == terms
    assert ix.terms() == list(terms.keys())  # fixture lists terms in lexicographic order


def test_token_dump_matches_hand_counted_buckets():
    docs, _, _ = load_corpus("corpus_edges.txt")
    text, off = gen.from_docs(docs)
    dump = oracle.dump_tokens(text, off)
    want_b = {b"42": 5, b"4x4": 0, b"80": 9, b"a\xc3\xb1o": 11, b"a\xc3\xb1os": 11, b"go": 17, b"x": 34, b"y": 35}
    assert [t for _, _, t in dump] == [b"go", b"go", b"go", b"42", b"4x4", b"80", b"a\xc3\xb1o", b"a\xc3\xb1o",
                                      b"a\xc3\xb1os", b"x", b"y", b"go", b"go"]
    assert [d for d, _, _ in dump] == [0, 0, 0, 0, 0, 0, 1, 1, 1, 3, 4, 5, 5]
    assert all(b == want_b[t] for _, b, t in dump)


# ---------------------------------------------------------------- brute force (library routines)
BYTE_POOL = list(b"aAbBzZ09 ,.-!\t\n") + [0x00, 0x7F, 0x80, 0xC3, 0xA9, 0xFF]


@settings(max_examples=150, deadline=None)
@given(st.lists(st.lists(st.sampled_from(BYTE_POOL), max_size=60).map(bytes), min_size=0, max_size=12))
def test_bruteforce_random(docs):
    ix = oracle_index(docs)
    want, n_tok, n_drop = brute_force(docs)
    assert ix.as_dict() == dict(sorted(want.items()))
    assert ix.n_tokens == n_tok and ix.n_dropped == n_drop and ix.n_docs == len(docs)


def test_length_boundary_255_256():
    docs = [b"x" * 255 + b" " + b"y" * 256 + b" " + b"Z" * 300, b"q" * 256 + b"Q"]
    ix = oracle_index(docs)
    assert ix.n_dropped == 3 and ix.n_tokens == 1
    assert ix.terms() == [b"x" * 255]


def test_generated_corpus_vs_bruteforce():
    text, off = gen.generate(gen.CONFIGS[1].scaled(vocab=2000))
    docs = [bytes(text[int(off[i]):int(off[i + 1])]) for i in range(len(off) - 1)]
    ix = oracle_index(docs)
    want, n_tok, n_drop = brute_force(docs)
    assert ix.as_dict() == dict(sorted(want.items()))
    assert (ix.n_tokens, ix.n_dropped) == (n_tok, n_drop)


# ---------------------------------------------------------------- coreutils
@pytest.mark.skipif(shutil.which("tr") is None or shutil.which("sort") is None, reason="coreutils")
def test_coreutils_dictionary_and_cf():
    text, off = gen.generate(gen.CONFIGS[1])
    docs = [bytes(text[int(off[i]):int(off[i + 1])]) for i in range(len(off) - 1)]
    # documents newline-separated so tokens never span documents (newline is a separator, S1)
    blob = b"\n".join(docs) + b"\n"
    cmd = ("LC_ALL=C tr -cs 'A-Za-z0-9\\200-\\377' '\\n' | LC_ALL=C tr A-Z a-z | "
           "LC_ALL=C awk 'length>0 && length<=255' | LC_ALL=C sort | LC_ALL=C uniq -c")
    out = subprocess.run(["bash", "-c", cmd], input=blob, capture_output=True, check=True).stdout
    want = []
    for line in out.splitlines():
        c, t = line.strip().split(b" ", 1)
        want.append((t, int(c)))
    ix = oracle_index(docs)
    got = list(zip(ix.terms(), ix.cf.tolist()))
    assert got == want


# ---------------------------------------------------------------- closed form
def test_closed_form_corpus():
    D, J = 600, 120
    text, off = gen.closed_form(D, J)
    ix = wjformat.parse(oracle.index_bytes(text, off))
    wjformat.check_invariants(ix)
    want = {}
    for j in range(J):
        docs = list(range(0, D, j + 1))
        assert len(docs) == -(-D // (j + 1))
        want[gen.closed_form_term(j)] = [(d, 1 + (d + j) % 3) for d in docs]
    assert len(set(want)) == J  # 7919 is coprime with 26 -> distinct terms
    assert ix.as_dict() == dict(sorted(want.items()))


# ---------------------------------------------------------------- metamorphic
def test_chunked_equals_single_and_mt():
    cfg = gen.CONFIGS[1].scaled(vocab=3000)
    text, off = gen.generate(cfg)
    single = oracle.index_bytes(text, off)
    o = oracle.Oracle()
    cuts = [0, 1, 1, 137, 500, 999, 1000]
    for a, b in zip(cuts, cuts[1:]):
        sub = off[a:b + 1] - off[a]
        o.add(text[int(off[a]):int(off[b])], sub)
    assert o.serialize() == single
    assert oracle.index_bytes(text, off, threads=4) == single


def test_concatenation_is_merge_with_offset():
    # partial postings of separate runs combine into the monolithic index.
    t1, o1 = gen.generate(gen.CONFIGS[1].scaled(vocab=500))
    a = wjformat.parse(oracle.index_bytes(t1[: int(o1[400])], o1[:401]))
    b = wjformat.parse(oracle.index_bytes(t1[int(o1[400]):], o1[400:] - o1[400]))
    full = wjformat.parse(oracle.index_bytes(t1, o1))
    merged = defaultdict(list)
    for t, p in a.as_dict().items():
        merged[t] += p
    for t, p in b.as_dict().items():
        merged[t] += [(d + 400, f) for d, f in p]
    assert full.as_dict() == dict(sorted(merged.items()))


def test_invariants_config1():
    text, off = gen.generate(gen.CONFIGS[1])
    ix = wjformat.parse(oracle.index_bytes(text, off))
    wjformat.check_invariants(ix)
    assert ix.n_docs == 1000 and ix.n_terms > 1000


# ---------------------------------------------------------------- f1: d-gap + variable-byte code
# Layout fixed by SURVEY.md §8(f1) ("7-bit groups, LSB-first, high bit = continuation"), the
# d-gaps by P:49, the encoding step by P:216; reading S19 in DESIGN.md.
VBYTE_TEXTBOOK = [(0, "00"), (1, "01"), (5, "05"), (127, "7f"), (128, "8001"), (300, "ac02"), (16383, "ff7f"),
                  (16384, "808001"), (2 ** 21, "80808001"), (2 ** 32 - 1, "ffffffff0f")]


@pytest.mark.parametrize("value,hexcode", VBYTE_TEXTBOOK)
def test_vbyte_hand_values(value, hexcode):
    assert oracle.vbyte([value]).hex() == hexcode


def test_vbyte_matches_protobuf_varint():
    # the same byte code is the protocol-buffers base-128 varint (library routine)
    enc = pytest.importorskip("google.protobuf.internal.encoder")
    rng = np.random.default_rng(7)
    vals = np.concatenate([rng.integers(0, 2 ** 32, 2000, dtype=np.uint64),
                           2 ** np.arange(32, dtype=np.uint64), 2 ** np.arange(1, 33, dtype=np.uint64) - 1])
    assert oracle.vbyte(vals.astype(np.uint32)) == b"".join(enc._VarintBytes(int(v)) for v in vals)


def test_vbyte_hand_counted_survey_corpus():
    # docs ["The cat sat.", "the CAT, the hat!", ""]: cat (0,1),(1,1); hat (1,1); sat (0,1);
    # the (0,1),(1,2) -> (gap, tf) bytes 00 01 01 01 | 01 01 | 00 01 | 00 01 01 02
    text, off = gen.from_docs([b"The cat sat.", b"the CAT, the hat!", b""])
    buf = oracle.index_bytes(text, off, vbyte=True)
    assert buf[:8] == b"WJINV002"
    hdr = np.frombuffer(buf, dtype="<u8", count=8)
    assert hdr[7] == 12
    assert buf[-16:-4] == bytes.fromhex("000101010101000100010102") and buf[-4:] == b"\0" * 4
    assert np.frombuffer(buf, dtype="<u8", count=5, offset=len(buf) - 16 - 40).tolist() == [0, 4, 6, 8, 12]


@pytest.mark.parametrize("which", ["config1", "edges", "bruteforce"])
def test_vbyte_decodes_to_pinned_index(which):
    if which == "config1":
        text, off = gen.generate(gen.CONFIGS[1])
    elif which == "edges":
        docs, _, _ = load_corpus("corpus_edges.txt")
        text, off = gen.from_docs(docs)
    else:
        rng = np.random.default_rng(3)
        docs = [bytes(rng.choice(BYTE_POOL, size=int(rng.integers(0, 80)))) for _ in range(300)]
        text, off = gen.from_docs(docs)
    plain = oracle.index_bytes(text, off)
    comp = oracle.index_bytes(text, off, vbyte=True)
    a, b = wjformat.parse(plain), wjformat.parse(comp)
    wjformat.check_invariants(b)
    for f in ("n_docs", "n_tokens", "n_dropped", "n_terms", "n_postings", "n_term_bytes"):
        assert getattr(a, f) == getattr(b, f)
    assert a.as_dict() == b.as_dict()
    assert len(comp) < len(plain) or a.n_postings == 0


# ---------------------------------------------------------------- f4: parser Steps 3-4
# Porter stemmer: the per-step examples printed in M.F. Porter, "An algorithm for suffix stripping"
# (Program 14(3), 1980), each applied to that step alone (step index 0..7 = 1a,1b,1c,2,3,4,5a,5b).
PORTER_STEP_EXAMPLES = {
    0: [("caresses", "caress"), ("ponies", "poni"), ("ties", "ti"), ("caress", "caress"), ("cats", "cat")],
    1: [("feed", "feed"), ("agreed", "agree"), ("plastered", "plaster"), ("bled", "bled"), ("motoring", "motor"),
        ("sing", "sing"), ("conflated", "conflate"), ("troubled", "trouble"), ("sized", "size"),
        ("hopping", "hop"), ("tanned", "tan"), ("falling", "fall"), ("hissing", "hiss"), ("fizzed", "fizz"),
        ("failing", "fail"), ("filing", "file")],
    2: [("happy", "happi"), ("sky", "sky")],
    3: [("relational", "relate"), ("conditional", "condition"), ("rational", "rational"), ("valenci", "valence"),
        ("hesitanci", "hesitance"), ("digitizer", "digitize"), ("conformabli", "conformable"),
        ("radicalli", "radical"), ("differentli", "different"), ("vileli", "vile"), ("analogousli", "analogous"),
        ("vietnamization", "vietnamize"), ("predication", "predicate"), ("operator", "operate"),
        ("feudalism", "feudal"), ("decisiveness", "decisive"), ("hopefulness", "hopeful"),
        ("callousness", "callous"), ("formaliti", "formal"), ("sensitiviti", "sensitive"),
        ("sensibiliti", "sensible")],
    4: [("triplicate", "triplic"), ("formative", "form"), ("formalize", "formal"), ("electriciti", "electric"),
        ("electrical", "electric"), ("hopeful", "hope"), ("goodness", "good")],
    5: [("revival", "reviv"), ("allowance", "allow"), ("inference", "infer"), ("airliner", "airlin"),
        ("gyroscopic", "gyroscop"), ("adjustable", "adjust"), ("defensible", "defens"), ("irritant", "irrit"),
        ("replacement", "replac"), ("adjustment", "adjust"), ("dependent", "depend"), ("adoption", "adopt"),
        ("homologou", "homolog"), ("communism", "commun"), ("activate", "activ"), ("angulariti", "angular"),
        ("homologous", "homolog"), ("effective", "effect"), ("bowdlerize", "bowdler")],
    6: [("probate", "probat"), ("rate", "rate"), ("cease", "ceas")],
    7: [("controll", "control"), ("roll", "roll")],
}


@pytest.mark.parametrize("step", sorted(PORTER_STEP_EXAMPLES))
def test_porter_paper_step_examples(step):
    for word, want in PORTER_STEP_EXAMPLES[step]:
        assert oracle.porter(word.encode(), step) == want.encode(), (step, word)


def test_porter_paper_whole_word_examples():
    # Porter's worked chains (GENERALIZATIONS -> ... -> GENER, OSCILLATORS -> ... -> OSCIL) and words
    # whose full result follows from the step examples above
    cases = {"generalizations": "gener", "oscillators": "oscil", "caresses": "caress", "ponies": "poni",
             "agreed": "agre", "relational": "relat", "rational": "ration", "conditional": "condit",
             "hopeful": "hope", "goodness": "good", "motoring": "motor", "plastered": "plaster",
             "replacement": "replac", "probate": "probat", "rate": "rate", "cease": "ceas", "controll": "control"}
    for word, want in cases.items():
        assert oracle.porter(word.encode()) == want.encode(), word
    # reading S20: fewer than 3 bytes, digits or bytes >= 0x80 -> unchanged
    for w in (b"is", b"as", b"3d", b"a\xc3\xb1os", b"abc1"):
        assert oracle.porter(w) == w


def test_stop_list_is_sklearn_english():
    text = pytest.importorskip("sklearn.feature_extraction.text")
    assert sorted(oracle.stop_words()) == sorted(text.ENGLISH_STOP_WORDS)


def test_stem_stop_hand_counted():
    # docs ["The cats sat.", "cat catS, the hat!", ""]; "the" is a stop word; cats -> cat
    text, off = gen.from_docs([b"The cats sat.", b"cat catS, the hat!", b""])
    ix = wjformat.parse(oracle.index_bytes(text, off, stem=True, stop=True))
    assert ix.as_dict() == {b"cat": [(0, 1), (1, 2)], b"hat": [(1, 1)], b"sat": [(0, 1)]}
    assert (ix.n_docs, ix.n_tokens, ix.n_dropped) == (3, 5, 0)
    # stop only: surface forms kept, "the" removed
    ix = wjformat.parse(oracle.index_bytes(text, off, stop=True))
    assert ix.as_dict() == {b"cat": [(1, 1)], b"cats": [(0, 1), (1, 1)], b"hat": [(1, 1)], b"sat": [(0, 1)]}


def test_stem_stop_invariants_and_chunking():
    text, off = gen.generate(gen.CONFIGS[1])
    one = oracle.index_bytes(text, off, stem=True, stop=True)
    ix = wjformat.parse(one)
    wjformat.check_invariants(ix)
    stems = set(ix.terms())
    o = oracle.Oracle(stem=True, stop=True)
    o.add(text[: int(off[500])], off[:501])
    o.add(text[int(off[500]):], off[500:] - off[500])
    assert o.serialize() == one
    assert oracle.index_bytes(text, off, threads=4, stem=True, stop=True) == one
    # every dictionary term is the stem of some token and none is a (stemmed) stop word
    stop = {oracle.porter(w.encode()) for w in oracle.stop_words()}
    assert not (stems & stop)
    surface = wjformat.parse(oracle.index_bytes(text, off))
    assert stems <= {oracle.porter(t) for t in surface.terms()}
