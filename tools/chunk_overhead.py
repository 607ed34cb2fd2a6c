"""Per-chunk fixed cost of the host pipeline: phase and kernel times for S = 1, 4, 8, 16 host chunks
of config 2 (device-timed per stream; phases overlap on the partials path)."""
import sys, time, numpy as np, torch
sys.path.insert(0, "/root/repo")
import gen, paper_conf_ipps_weij11_b200 as wj
text, off = gen.generate(gen.CONFIGS[2])
th = torch.from_numpy(text).pin_memory()
T = len(text); nd = len(off) - 1
for S in [1, 4, 8, 16]:
    cuts = sorted({0, nd} | {int(np.searchsorted(off, T * k // S)) for k in range(1, S)})
    parts = [(th[int(off[a]):int(off[b])], torch.from_numpy((off[a:b + 1] - off[a]).astype(np.int64)).pin_memory())
             for a, b in zip(cuts, cuts[1:])]
    ix = wj.Index(profile=True, pipeline=True)
    def run():
        torch.cuda.synchronize(); t0 = time.time()
        ix.reset()
        for t, o in parts:
            ix.add_stream(t, o)
        ix.finalize(); torch.cuda.synchronize()
        return time.time() - t0
    for it in range(3):
        run()
    a = ix.stats(); dt = run(); b = ix.stats()
    d = lambda k: {n: round(b[k][n] - a[k][n], 2) for n in b[k] if b[k][n] != a[k][n]}
    print("S", S, "add+finalize ms", round(dt * 1e3, 2), "syncs", b["host_syncs"] - a["host_syncs"], flush=True)
    print("  phase_ms", d("phase_ms"), flush=True)
    print("  kernel_ms", d("kernel_ms"), flush=True)
    ix.close()
