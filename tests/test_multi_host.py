"""Multi-GPU host-side logic on CPU (no GPU): the owner map, the K-way merge of
per-rank dictionary slices done by the C ABI (index_merge_serialized), and the torch.distributed
(gloo, world_size 2) gather + merge protocol that bench.py uses for N > 1."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import gen
import oracle
import paper_conf_ipps_weij11_b200 as wj
import wjformat


def test_owner_map_paper_example():
    # "if unpopular trie collections have indices (0, 13, 27, 175, 384, 5810, 10041, 17316) and there
    # are two GPU, then (0, 384, 5810, 17316) are assigned to GPU indexer 0 and (13, 27, 175, 10041) to GPU 1"
    idx = [0, 13, 27, 175, 384, 5810, 10041, 17316]
    assert [i for i in idx if wj.owner_of(i, 2) == 0] == [0, 384, 5810, 17316]
    assert [i for i in idx if wj.owner_of(i, 2) == 1] == [13, 27, 175, 10041]


def test_serialize_helper_roundtrip():
    text, off = gen.generate(gen.CONFIGS[1].scaled(vocab=500))
    b = oracle.index_bytes(text, off)
    ix = wjformat.parse(b)
    d = ix.as_dict()
    assert wjformat.serialize(ix.n_docs, ix.n_tokens, ix.n_dropped, ix.terms(), [d[t] for t in ix.terms()]) == b


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_merge_of_owner_slices_is_the_global_index(world):
    text, off = gen.generate(gen.CONFIGS[1])
    full = oracle.index_bytes(text, off)
    slices = wjformat.split_by_owner(full, world, oracle.bucket)
    assert wj.merge_serialized(slices) == full


def test_merge_rejects_bad_input():
    text, off = gen.from_docs([b"a b", b"c"])
    good = oracle.index_bytes(text, off)
    with pytest.raises(wj.WJError):
        wj.merge_serialized([good, b"not an index"])
    t2, o2 = gen.from_docs([b"a b"])
    with pytest.raises(wj.WJError):  # slices must agree on n_docs
        wj.merge_serialized([good, oracle.index_bytes(t2, o2)])


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _gloo_worker(rank, world, port, q):
    import torch.distributed as dist

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    text, off = gen.generate(gen.CONFIGS[1])
    full = oracle.index_bytes(text, off)
    mine = wjformat.split_by_owner(full, world, oracle.bucket)[rank]  # this rank's dictionary slice
    got = [None] * world
    dist.all_gather_object(got, mine)
    if rank == 0:
        q.put(wj.merge_serialized(got) == full)
    dist.destroy_process_group()


def test_gloo_world2_gather_and_merge():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_gloo_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    ok = q.get(timeout=120)
    for p in ps:
        p.join(timeout=60)
    assert ok


# ---------------------------------------------------------------- balanced owner map (host)
def test_balance_owners_lpt_properties():
    wj = pytest.importorskip("paper_conf_ipps_weij11_b200")
    rng = np.random.default_rng(5)
    counts = np.zeros(17613, dtype=np.uint64)
    nz = rng.choice(17613, 6000, replace=False)
    counts[nz] = (1e6 / np.arange(1, 6001) ** 1.1).astype(np.uint64) + 1  # Zipf-like collection sizes
    for K in (2, 3, 4, 8):
        own = wj.balance_owners(counts, K)
        assert own.max() < K
        zero = counts == 0
        assert np.array_equal(own[zero], np.arange(17613)[zero] % K)  # unsampled: b mod K
        load = np.bincount(own, weights=counts.astype(np.float64), minlength=K)
        # greedy LPT: the busiest rank exceeds the mean by at most the largest single item
        assert load.max() <= load.sum() / K + counts.max()
        mod = np.bincount(np.arange(17613) % K, weights=counts.astype(np.float64), minlength=K)
        assert load.max() <= mod.max()
    # hand example: counts 5,4,3,3,3 over 2 ranks -> 5->r0, 4->r1, 3->r1 (4<5), 3->r0 (8>7? r0=5<7), 3->r1
    own = wj.balance_owners(np.array([5, 4, 3, 3, 3], dtype=np.uint64), 2)
    assert own.tolist() == [0, 1, 1, 0, 1]


def _gloo_owner_map_worker(rank, world, port, q):
    """The balanced owner map protocol of the multi-rank path (engine.cu build_owner_map):
    each rank counts the tokens per trie collection of its own document range (the oracle's token dump
    stands in for the device sample), the counts are all-gathered (gloo here, NCCL in the library), and
    every rank bin-packs the summed counts with the library's host LPT (index_balance_owners)."""
    import torch.distributed as dist

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    text, off = gen.generate(gen.CONFIGS[1].scaled(vocab=3000))
    n = len(off) - 1
    lo, hi = n * rank // world, n * (rank + 1) // world
    t = text[int(off[lo]):int(off[hi])]
    o = (np.asarray(off[lo:hi + 1], dtype=np.uint64) - off[lo]).astype(np.uint64)
    counts = np.zeros(wj.N_COLLECTIONS, dtype=np.uint64)
    for _, b, _ in oracle.dump_tokens(t, o):
        counts[b] += 1
    allc = [None] * world
    dist.all_gather_object(allc, counts)
    own = wj.balance_owners(np.sum(allc, axis=0).astype(np.uint64), world)
    maps = [None] * world
    dist.all_gather_object(maps, own)
    full = oracle.index_bytes(text, off)
    mine = wjformat.split_by_owner(full, world, lambda term: int(own[oracle.bucket(term)]))[rank]
    got = [None] * world
    dist.all_gather_object(got, mine)
    if rank == 0:
        q.put(all(np.array_equal(maps[0], m) for m in maps) and wj.merge_serialized(got) == full
              and not np.array_equal(own, np.arange(wj.N_COLLECTIONS) % world))
    dist.destroy_process_group()


def test_gloo_world2_balanced_owner_map_protocol():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_gloo_owner_map_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    ok = q.get(timeout=180)
    for p in ps:
        p.join(timeout=60)
    assert ok
