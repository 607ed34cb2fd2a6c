import sys, time, numpy as np, torch
sys.path.insert(0, "/root/repo")
import gen, paper_conf_ipps_weij11_b200 as wj
text, off = gen.generate(gen.CONFIGS[2])
th = torch.from_numpy(text).pin_memory()
for S, vb in [(8, True), (8, False), (4, True)]:
    T = len(text); nd = len(off) - 1
    cuts = sorted({0, nd} | {int(np.searchsorted(off, T * k // S)) for k in range(1, S)})
    parts = [(th[int(off[a]):int(off[b])], torch.from_numpy((off[a:b + 1] - off[a]).astype(np.int64)).pin_memory())
             for a, b in zip(cuts, cuts[1:])]
    ix = wj.Index(profile=True, vbyte=vb, pipeline=True)
    for it in range(4):
        t0 = time.time()
        ix.reset()
        ts = []
        for t, o in parts:
            ix.add_stream(t, o); ts.append(time.time() - t0)
        ix.finalize(); t1 = time.time() - t0
        n = ix.serialized_size()
        out = torch.empty(n, dtype=torch.uint8, pin_memory=True)
        ix.serialize_into(out.data_ptr(), n); t2 = time.time() - t0
        st = ix.stats()
        print(S, vb, it, [round(x * 1e3, 1) for x in ts], round(t1 * 1e3, 1), round(t2 * 1e3, 1), st["device_bytes"] >> 20, st["host_syncs"], flush=True)
    ph = ix.stats()["phase_ms"]
    print({k: round(v, 1) for k, v in ph.items() if v})
    ix.close()
