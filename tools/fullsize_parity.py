"""Full-size parity of BASELINE.json configs (SURVEY §8(c) bar: byte-identical serialized index).

Test infrastructure (calls oracle/): every chunk of the config is generated on the host, indexed by the
CUDA path from device memory (one index_add_stream per 1 GiB chunk, as the paper's runs), and
added to the doc-range-sharded CPU oracle (oracle_add_mt); the two serialized files are compared by
SHA-256 and the invariants of tests/wjformat.py are checked on the GPU's file.

usage (GPU box): python tools/fullsize_parity.py --configs 3 4 [--chunks K] [--out gpurun_out/fullsize.json]
"""
import argparse
import hashlib
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path[:0] = [ROOT, os.path.join(ROOT, "tests")]
import gen  # noqa: E402
import oracle  # noqa: E402
import wjformat  # noqa: E402
import paper_conf_ipps_weij11_b200 as wj  # noqa: E402


def run(cfg_id: int, chunks: int | None, threads: int, invariants: bool = True) -> dict:
    cfg = gen.CONFIGS[cfg_id]
    n_chunks = chunks or cfg.chunks
    o = oracle.Oracle()
    t_gpu = t_orc = t_gen = 0.0
    total = 0
    with wj.Index(device=0) as ix:
        for c in range(n_chunks):
            t0 = time.time()
            text, off = gen.generate(cfg, c, threads=threads)
            t_gen += time.time() - t0
            total += text.size
            tt = torch.from_numpy(text).cuda()
            to = torch.from_numpy(off.astype(np.int64)).cuda()
            torch.cuda.synchronize()
            t0 = time.time()
            ix.add_stream(tt, to)
            torch.cuda.synchronize()
            t_gpu += time.time() - t0
            del tt, to
            t0 = time.time()
            o.add(text, off, threads)
            t_orc += time.time() - t0
        t0 = time.time()
        ix.finalize()
        got = ix.serialize()
        t_gpu += time.time() - t0
        st = ix.stats()
    t0 = time.time()
    want = o.serialize()
    t_orc += time.time() - t0
    hg, hw = hashlib.sha256(got).hexdigest(), hashlib.sha256(want).hexdigest()
    f = wjformat.parse(got)
    if invariants:  # numpy copies of every array: skipped for the largest runs (host memory)
        wjformat.check_invariants(f)
    return {"config": cfg_id, "workload": cfg.name, "chunks": n_chunks, "bytes": total,
            "n_docs": f.n_docs, "n_tokens": f.n_tokens, "n_terms": f.n_terms, "n_postings": f.n_postings,
            "serialized_bytes": len(got), "sha256_gpu": hg, "sha256_oracle": hw, "identical": got == want,
            "gpu_wall_s": round(t_gpu, 2), "oracle_wall_s": round(t_orc, 2), "gen_wall_s": round(t_gen, 2),
            "oracle_threads": threads, "btree_height_max": st["btree_height_max"], "invariants_checked": invariants}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", type=int, nargs="+", default=[3, 4])
    ap.add_argument("--chunks", type=int, default=None, help="first K chunks only (e.g. a config-5 prefix)")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "fullsize.json"))
    ap.add_argument("--no-invariants", action="store_true", help="SHA-256 comparison only")
    a = ap.parse_args()
    threads = max(1, len(os.sched_getaffinity(0)))
    res = []
    for c in a.configs:
        r = run(c, a.chunks, threads, not a.no_invariants)
        print(json.dumps(r), flush=True)
        res.append(r)
        with open(a.out, "w") as f:
            json.dump(res, f, indent=1)
    sys.exit(0 if all(r["identical"] for r in res) else 1)


if __name__ == "__main__":
    main()
