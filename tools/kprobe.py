"""Per-kernel times of the single-GPU path on config-2-shaped corpora of several vocabulary sizes
(diagnostic: separates table-miss cost from per-token instruction cost).
usage: python tools/kprobe.py [vocab ...]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_weij11_b200 as wj  # noqa: E402

vocabs = [int(x) for x in sys.argv[1:]] or [10_000, 5_000_000]
for v in vocabs:
    text, off = gen.generate(gen.CONFIGS[2].scaled(vocab=v))
    td = torch.from_numpy(text).cuda()
    od = torch.from_numpy(off.astype(np.int64)).cuda()
    ix = wj.Index(device=0, profile=True)
    for _ in range(2):
        ix.reset(); ix.add_stream(td, od); ix.finalize()
    torch.cuda.synchronize()
    s0 = ix.stats()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    K = 5
    e0.record()
    for _ in range(K):
        ix.reset(); ix.add_stream(td, od); ix.finalize()
    e1.record()
    torch.cuda.synchronize()
    s1 = ix.stats()
    ks = " ".join(f"{k}={(s1['kernel_ms'][k] - s0['kernel_ms'][k]) / K:.3f}" for k in wj.KERNELS
                  if s1['kernel_count'][k] > s0['kernel_count'][k])
    ph = " ".join(f"{k}={(s1['phase_ms'][k] - s0['phase_ms'][k]) / K:.3f}" for k in s1["phase_ms"]
                  if s1['phase_ms'][k] > s0['phase_ms'][k])
    print(f"V={v} N={s1['n_tokens']} terms={s1['n_terms']} ms={e0.elapsed_time(e1) / K:.3f} | {ks} | {ph}", flush=True)
    ix.close()
