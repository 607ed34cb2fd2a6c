"""Concurrency timeline of one config-2 step (torch.profiler / CUPTI, kernels on every stream of the
process, including libwjindex.so's): prints each kernel's start / end (ms from the step start) per stream,
and per-stream busy time.  usage: python tools/trace_step.py [--profile-flag] > trace.txt"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_ipps_weij11_b200 as wj  # noqa: E402

prof_flag = "--profile-flag" in sys.argv
text, doc_off = bench.corpus(2, 0, None)
text_d = torch.from_numpy(text).cuda()
off_d = torch.from_numpy(doc_off.astype(np.int64)).cuda()
ix = wj.Index(device=0, profile=prof_flag)


def step():
    ix.reset()
    ix.add_stream(text_d, off_d)
    ix.finalize()


for _ in range(4):
    step()
torch.cuda.synchronize()
from torch.profiler import ProfilerActivity, profile  # noqa: E402

with profile(activities=[ProfilerActivity.CUDA]) as p:
    step()
    torch.cuda.synchronize()
p.export_chrome_trace("/tmp/trace.json")
ev = [e for e in json.load(open("/tmp/trace.json"))["traceEvents"]
      if e.get("ph") == "X" and e.get("cat") in ("kernel", "gpu_memset", "gpu_memcpy")]
t0 = min(e["ts"] for e in ev)
ev.sort(key=lambda e: e["ts"])
streams = sorted({e["args"].get("stream", e.get("tid")) for e in ev})
busy = {s: 0.0 for s in streams}
for e in ev:
    s = e["args"].get("stream", e.get("tid"))
    busy[s] += e["dur"] / 1000
    name = e["name"].replace("void ", "").replace("wj::", "")[:70]
    print(f"{(e['ts'] - t0) / 1000:8.3f} {(e['ts'] + e['dur'] - t0) / 1000:8.3f} s{streams.index(s)} {name}")
end = max(e["ts"] + e["dur"] for e in ev)
print(f"step span {(end - t0) / 1000:.3f} ms; busy per stream:", {f"s{streams.index(s)}": round(v, 3) for s, v in busy.items()})
