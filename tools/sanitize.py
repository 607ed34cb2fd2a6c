"""Small end-to-end runs for compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
config 1 on one GPU (per-run partial lists: side + dictionary streams, event joins), the host
pipeline (copy stream), hot-term matrix, the global-stream path, and the loopback transport at
K = 2 (two contexts, two host threads).  Each run is checked against the CPU oracle.
usage: compute-sanitizer --tool memcheck python tools/sanitize.py [--small]"""
import os
import sys
import threading

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_weij11_b200 as wj  # noqa: E402

text, off = gen.generate(gen.CONFIGS[1])
off = np.asarray(off, dtype=np.uint64)
if "--small" in sys.argv:  # racecheck is ~100x slower: the first 160 documents of config 1
    text, off = text[: int(off[160])], off[:161]
want = oracle.index_bytes(text, off)
n = len(off) - 1
cuts = [0, n * 3 // 10, n * 3 // 10 + 1, n]


def run(**kw):
    with wj.Index(device=0, **kw) as ix:
        for a, b in zip(cuts, cuts[1:]):
            ix.add_stream(text[int(off[a]):int(off[b])].copy(), off[a:b + 1] - off[a])
        ix.finalize()
        got = ix.serialize()
    assert got == want, kw
    print("ok", kw, flush=True)


run()
run(pipeline=True)
run(hot=True)
run(global_stream=True)
run(vbyte=False, profile=True)

K = 2
hub = wj.LoopbackHub(K)
slices = [None] * K


def rank(r):
    with wj.Index(device=0, rank=r, world=K, hub=hub, own_stream=True) as ix:
        for a, b in zip(cuts, cuts[1:]):
            bounds = [a + (b - a) * i // K for i in range(K + 1)]
            lo, hi = bounds[r], bounds[r + 1]
            ix.add_stream(text[int(off[lo]):int(off[hi])].copy(), off[lo:hi + 1] - off[lo])
        ix.finalize()
        slices[r] = ix.serialize()


th = [threading.Thread(target=rank, args=(r,)) for r in range(K)]
for t in th:
    t.start()
for t in th:
    t.join()
hub.close()
assert wj.merge_serialized(slices) == want
print("ok loopback K=2", flush=True)
print("SANITIZE_DONE")
