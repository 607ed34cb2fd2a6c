#!/usr/bin/env python
"""Benchmark: indexing throughput of the B200 indexer on BASELINE.json configs[1]
(ClueWeb09-shaped synthetic, 1 GiB of raw text per GPU).

One step = one pass of the whole hot path over one batch: index_reset + index_add_stream (1 GiB,
device-resident) + index_finalize (the final inverted file on the device).  Timed with CUDA events
on the stream the library launches on, after W warm-up steps, bracketed by barrier + synchronize,
max over ranks.  Inputs (1 GiB) are larger than L2 (126 MB), so no L2 flush is needed.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config 2]

N > 1 (torchrun): every rank submits its own 1 GiB document range (chunk index = rank; rank order =
DocID order) and the library routes each term to the rank owning its trie collection (b mod N,
PAPER.md P:210) with an NCCL all-to-all-v over NVLink; each rank builds its exclusive dictionary
slice.  Per-GPU work is fixed as N grows: scaling is weak.  ``--impl reference`` times the CPU oracle (the reference arm of
this tier) on a bounded document prefix of the same workload, on rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import gen  # noqa: E402

METRIC = "indexing throughput, MB/s of raw text (1 MB = 10^6 B)"
WORKLOAD = {2: "clueweb09-shaped synthetic, 1 GiB per GPU (BASELINE configs[1])"}
HBM_FALLBACK_GBS = 6650.0

# Algorithmic bytes per launch of each timed kernel, given the chunk's
# T (text bytes), N (kept tokens), P (postings), E (stream elements after the per-document combine).
KERNEL_BYTES = {
    "tokenize_count": lambda T, N, P, E: T,                 # read the text once
    "tokenize_emit": lambda T, N, P, E: T + 8 * N,          # read text, write (slot u32, doc u32) per token
    "slot_to_tid": lambda T, N, P, E: 8 * N,                # read + write u32 per token
    "map_rank": lambda T, N, P, E: 8 * E,                   # read + write u32 per element
    "sort_hist": lambda T, N, P, E: 4 * E,                  # read u32 keys
    "sort_scatter": lambda T, N, P, E: 16 * E,              # read + write (u32 key, u32 doc) per element
    "rle_emit": lambda T, N, P, E: 8 * E + 8 * P,           # read (key, doc), write (docid, tf)
    "copy_partials": lambda T, N, P, E: 16 * P,             # read + write (docid, tf) per posting
}


def measured_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy bandwidth)"
    except Exception:
        return HBM_FALLBACK_GBS, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.device = device
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "50"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 8:
                continue
            try:
                sm.append(float(parts[0]))
                smax.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def corpus(cfg_id: int, chunk: int, chunk_bytes: int | None = None):
    cfg = gen.CONFIGS[cfg_id]
    if chunk_bytes is not None:
        cfg = cfg.scaled(chunk_bytes=chunk_bytes)
    return gen.generate(cfg, chunk=chunk)


def cpu_baseline(text, doc_off, trials: int = 3, st_target_s: float = 4.0, mt_budget_s: float = 45.0):
    """The CPU oracle as it stands (never tuned), BASELINE.md's plan: oracle_st (one thread, pinned to
    one core) on a bounded document prefix, and oracle_mt (contiguous document ranges over all host
    cores, per-term lists concatenated in range order) on the whole workload; `trials` timed runs
    each (3 trials), mean and (max - min) / mean spread."""
    import oracle

    cores = len(os.sched_getaffinity(0))

    def run(nbytes, threads):
        nd = int(np.searchsorted(doc_off, nbytes, side="right")) - 1
        nd = max(1, min(nd, len(doc_off) - 1))
        t0 = time.perf_counter()
        o = oracle.Oracle()
        o.add(text[: int(doc_off[nd])], doc_off[: nd + 1], threads=threads)
        o.serialize()
        o.close()
        return int(doc_off[nd]), nd, time.perf_counter() - t0

    def stats(vals):
        m = sum(vals) / len(vals)
        return m, (max(vals) - min(vals)) / m if m else 0.0

    aff = os.sched_getaffinity(0)
    try:
        os.sched_setaffinity(0, {min(aff)})  # oracle_st pinned to one core (taskset -c analogue)
        b, nd, dt = run(2 << 20, 1)
        want = int(min(len(text), max(b, b / max(dt, 1e-6) * st_target_s)))
        st = [run(want, 1) for _ in range(trials)]
    finally:
        os.sched_setaffinity(0, aff)
    st_b, st_nd = st[0][0], st[0][1]
    st_mean, st_spread = stats([x[0] / x[2] / 1e6 for x in st])
    # oracle_mt on the whole workload if one run fits ~25 s of wall time, else on a document prefix
    b, nd, dt = run(min(len(text), 32 << 20), cores)
    mt_bytes = int(min(len(text), max(b, b / max(dt, 1e-6) * 25.0)))
    mt, spent = [], 0.0
    for _ in range(trials):
        r = run(mt_bytes, cores)
        mt.append(r)
        spent += r[2]
        if spent > mt_budget_s:
            break
    mt_mean, mt_spread = stats([x[0] / x[2] / 1e6 for x in mt])
    return {"value": mt_mean, "unit": "MB/s", "cores": cores, "kind": "oracle",
            "sample": (f"oracle_mt: first {mt[0][1]} of {len(doc_off) - 1} documents ({mt[0][0]} of {len(text)} B), {cores} "
                       f"threads over contiguous document ranges, oracle_add + serialize, {len(mt)} trial(s); "
                       f"oracle_st: first {st_nd} documents ({st_b} B), 1 thread pinned to one core, {trials} trials"),
            "trials": len(mt), "spread": mt_spread,
            "st": {"value": st_mean, "unit": "MB/s", "cores": 1, "trials": trials, "spread": st_spread,
                   "sample_bytes": st_b},
            "mt": {"value": mt_mean, "unit": "MB/s", "cores": cores, "trials": len(mt), "spread": mt_spread,
                   "sample_bytes": mt[0][0], "seconds": [round(x[2], 3) for x in mt]}}


def run_reference(args, rank, world):
    """Reference arm of this tier: the CPU oracle as it stands (oracle_mt over all host cores) on a
    bounded document prefix of the same workload, sized so that warmup + steps finish in ~2.5 min."""
    if rank != 0:
        return
    import oracle

    cores = len(os.sched_getaffinity(0))
    text, doc_off = corpus(args.config, 0, args.chunk_bytes)

    def prefix(nbytes):
        nd = int(np.searchsorted(doc_off, nbytes, side="right")) - 1
        nd = max(1, min(nd, len(doc_off) - 1))
        return text[: int(doc_off[nd])], doc_off[: nd + 1]

    def step(t, o):
        x = oracle.Oracle()
        x.add(t, o, threads=cores)
        x.serialize()
        x.close()

    t, o = prefix(64 << 20)
    t0 = time.perf_counter()
    step(t, o)
    rate = len(t) / max(time.perf_counter() - t0, 1e-6)
    budget = 150.0 / max(1, args.steps + args.warmup)
    t, o = prefix(int(min(len(text), max(len(t), rate * budget))))
    nd = len(o) - 1
    for _ in range(args.warmup):
        step(t, o)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        step(t, o)
        times.append(time.perf_counter() - t0)
    dt = sum(times) / len(times)
    val = len(t) / dt / 1e6
    sample = (f"first {nd} documents ({len(t)} B) of the same corpus per step, oracle_mt (std::map per "
              f"contiguous document range, {cores} threads) + serialize")
    line = {
        "impl": "reference", "metric": METRIC, "value": val, "unit": "MB/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": WORKLOAD.get(args.config, str(args.config)), "sample": sample},
        "cpu_baseline": {"value": val, "unit": "MB/s", "cores": cores, "kind": "oracle", "sample": sample,
                         "spread": (max(times) - min(times)) / dt if dt else 0.0},
        "e2e": {"value": val, "unit": "MB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print_json(line)


def steady_state(wj, ix, args, device):
    """Multi-chunk leg (N = 1): S device-resident 1 GiB chunks of config 5 per step (reset + S x
    add_stream + finalize), so every chunk after the first probes and extends a non-empty dictionary
    ("Fig. 11").  Reports MB/s, ms per chunk and the per-kernel / per-phase ms per chunk."""
    import torch

    S = args.steady_chunks
    parts = []
    for c in range(S):
        t, o = corpus(5, c)
        parts.append((torch.from_numpy(t).cuda(), torch.from_numpy(o.astype(np.int64)).cuda(), len(t)))
    T = sum(p[2] for p in parts)

    def step():
        ix.reset()
        for t, o, _ in parts:
            ix.add_stream(t, o)
        ix.finalize()

    step()
    torch.cuda.synchronize()
    s0 = ix.stats()
    steps = 3
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps):
        step()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    s1 = ix.stats()
    kms = {k: round((s1["kernel_ms"][k] - s0["kernel_ms"][k]) / steps / S, 4) for k in wj.KERNELS
           if s1["kernel_count"][k] > s0["kernel_count"][k]}
    pms = {k: round((s1["phase_ms"][k] - s0["phase_ms"][k]) / steps / S, 4) for k in wj.PHASES
           if s1["phase_ms"][k] > s0["phase_ms"][k]}
    b_min = T + 8 * s1["n_postings"] + s1["n_term_bytes"] + 28 * s1["n_terms"]
    peak, _ = measured_peak()
    del parts
    torch.cuda.empty_cache()
    return {"workload": f"config 5 (ClueWeb09-shaped) prefix: {S} x 1 GiB chunks, device-resident", "chunks": S,
            "bytes": T, "ms_per_step": ms, "ms_per_chunk": ms / S, "value": T / (ms / 1e3) / 1e6, "unit": "MB/s",
            "n_terms": s1["n_terms"], "n_postings": s1["n_postings"], "n_tokens": s1["n_tokens"],
            "btree_height_max": s1["btree_height_max"], "new_terms_last_chunk": s1["new_terms_last"],
            "roofline_frac": b_min / (ms / 1e3) / 1e9 / peak, "steps": steps,
            "kernels_ms_per_chunk": kms, "phases_ms_per_chunk": pms,
            "host_syncs_per_chunk": (s1["host_syncs"] - s0["host_syncs"]) / steps / S,
            "launches_per_chunk": (s1["kernel_launches"] - s0["kernel_launches"]) / steps / S}


def print_json(obj):  # replaced in main() by a writer bound to the real stdout
    print(json.dumps(obj), flush=True)


def main():
    # The driver parses exactly one JSON line from stdout: keep the real stdout for it and send
    # everything else (NCCL's version banner, library prints) to stderr.
    json_out = os.fdopen(os.dup(1), "w")
    sys.stdout.flush()
    os.dup2(2, 1)
    global print_json
    print_json = lambda obj: (json_out.write(json.dumps(obj) + "\n"), json_out.flush())  # noqa: E731
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--chunk-bytes", type=int, default=None, help="override bytes per GPU (debug)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--e2e-chunks", type=int, default=4,
                    help="e2e: feed the step as this many pinned host chunks through the host pipeline")
    ap.add_argument("--steady-chunks", type=int, default=4,
                    help="multi-chunk leg: this many 1 GiB chunks of config 5 (ClueWeb scale, SURVEY 8(d)) per step, "
                         "device-resident, so the B-tree probe, merge and rebuild run on a non-empty dictionary (0: off)")
    ap.add_argument("--hot", action="store_true", help="sampled hot-term aggregation (SURVEY 8(f2)(ii), opt-in)")
    ap.add_argument("--vbyte", action="store_true",
                    help="also encode the postings as d-gaps + variable-byte code (SURVEY 8(f1), WJINV002)")
    args = ap.parse_args()
    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))

    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    import torch.distributed as dist

    import paper_conf_ipps_weij11_b200 as wj

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    text, doc_off = corpus(args.config, rank, args.chunk_bytes)
    T = len(text)
    text_h = torch.from_numpy(text).pin_memory()
    off_h = torch.from_numpy(doc_off.astype(np.int64)).pin_memory()
    text_d = text_h.cuda()
    off_d = off_h.cuda()
    torch.cuda.synchronize()

    hot = args.hot
    force_dist = os.environ.get("WJ_BENCH_FORCE_DIST") == "1"  # exercise the NCCL path at N=1
    if world > 1 or force_dist:
        nid = [wj.nccl_unique_id() if rank == 0 else None]
        if world > 1:
            dist.broadcast_object_list(nid, src=0)
        ix = wj.Index(device=local, profile=False, rank=rank, world=world, nccl_id=nid[0], vbyte=args.vbyte,
                      balanced=world > 1)
    else:
        # the timed context records no per-phase / per-kernel events (that instrumentation adds event
        # records and host-side event queries to every step); the breakdown comes from a second,
        # profiled context below
        ix = wj.Index(device=local, profile=False, vbyte=args.vbyte, hot=hot)

    def step(t, o):
        ix.reset()
        ix.add_stream(t, o)
        ix.finalize()

    for _ in range(args.warmup):
        step(text_d, off_d)
    torch.cuda.synchronize()
    s0 = ix.stats()
    N, P, V = s0["n_tokens"], s0["n_postings"], s0["n_terms"]

    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.15)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(args.steps):
        step(text_d, off_d)
    e1.record()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    ms = e0.elapsed_time(e1) / args.steps
    s1 = ix.stats()
    if world > 1:
        t = torch.tensor([ms], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())

    total_bytes = T * world
    value = total_bytes / (ms / 1e3) / 1e6
    launches = (s1["kernel_launches"] - s0["kernel_launches"]) / args.steps

    # per-phase / per-kernel breakdown: a profiled context (CUDA events around phases and kernels) run on
    # the same input for a few steps after the timed ones
    prof_steps = max(1, min(args.steps, 5))
    if world > 1 or force_dist:
        nidp = [wj.nccl_unique_id() if rank == 0 else None]
        if world > 1:
            dist.broadcast_object_list(nidp, src=0)
        ixp = wj.Index(device=local, profile=True, rank=rank, world=world, nccl_id=nidp[0], vbyte=args.vbyte,
                       balanced=world > 1)
    else:
        ixp = wj.Index(device=local, profile=True, vbyte=args.vbyte, hot=hot)

    def pstep():
        ixp.reset()
        ixp.add_stream(text_d, off_d)
        ixp.finalize()

    for _ in range(max(2, args.warmup)):  # (its buffers grow to the steady sizes first)
        pstep()
    torch.cuda.synchronize()
    p0 = ixp.stats()
    for _ in range(prof_steps):
        pstep()
    torch.cuda.synchronize()
    p1 = ixp.stats()

    # per-kernel efficiency of the dominant timed kernel on its own implementation bytes (design
    # evidence only: SURVEY 8(d) excludes implementation bytes from the headline)
    peak, peak_src = measured_peak()
    kms = {k: p1["kernel_ms"][k] - p0["kernel_ms"][k] for k in wj.KERNELS}
    kcnt = {k: p1["kernel_count"][k] - p0["kernel_count"][k] for k in wj.KERNELS}
    dom = max((k for k in KERNEL_BYTES if kcnt.get(k)), key=lambda k: kms[k])
    per_launch_ms = kms[dom] / kcnt[dom]
    E = s1["stream_elems"]
    bytes_per_launch = KERNEL_BYTES[dom](T, N, P, E)
    achieved = bytes_per_launch / (per_launch_ms / 1e3) / 1e9
    # headline roofline = SURVEY 8(d): compulsory bytes B_min = T + 8P + sum(len + 28) over terms of
    # the step, over the step time, against the measured HBM copy bandwidth
    post_bytes = 8 * P
    if args.vbyte:  # compressed postings: the code bytes replace the (docid, tf) arrays
        pad8 = lambda x: (x + 7) & ~7  # noqa: E731
        post_bytes = ix.serialized_size() - (64 + 16 * (V + 1) + pad8(s1["n_term_bytes"]) + pad8(4 * V) + 8 * V)
    b_min = T + post_bytes + s1["n_term_bytes"] + 28 * V
    step_gbs = b_min * world / (ms / 1e3) / 1e9
    traffic = None
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tp) and args.config == 2 and world == 1 and not args.vbyte:
        try:
            traffic = json.load(open(tp)).get("step_dram_bytes")
        except Exception:
            traffic = None

    phases = {k: (p1["phase_ms"][k] - p0["phase_ms"][k]) / prof_steps for k in wj.PHASES}
    # all-to-all-v rounds of the multi-rank path: bytes this rank sent per step, device-
    # synchronised wall time of the rounds, fraction of 900 GB/s per direction (NVLink 5), max over ranks
    xb = (s1["exchange_bytes"] - s0["exchange_bytes"]) / args.steps
    xms = (s1["exchange_ms"] - s0["exchange_ms"]) / args.steps
    if world > 1:
        t = torch.tensor([xb, xms], device="cuda", dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        xb, xms = float(t[0].item()), float(t[1].item())
    exchange = {"bytes_per_step": xb, "ms_per_step": xms,
                "nvlink_frac": (xb / (xms / 1e3) / 900e9) if xms > 0 and xb > 0 else None,
                "bytes_per_gib_text": xb / (T / 2**30)}
    kernels = {k: {"ms_per_step": kms[k] / prof_steps, "launches_per_step": kcnt[k] / prof_steps} for k in wj.KERNELS}

    # e2e through the public API with host buffers: H2D of the chunk inside, D2H of the whole index.
    # --e2e-chunks S > 1 feeds the step's text as S pinned host chunks to a context with the host
    # pipeline (Fig. 9: the copy of chunk c+1 overlaps the indexing of chunk c).
    def e2e_leg(vbyte):
        S = max(1, args.e2e_chunks)
        nid2 = [None]
        if world > 1 or force_dist:  # a fresh communicator for the second context
            nid2 = [wj.nccl_unique_id() if rank == 0 else None]
            if world > 1:
                dist.broadcast_object_list(nid2, src=0)
        ixe = wj.Index(device=local, rank=rank, world=world, vbyte=vbyte, pipeline=S > 1, nccl_id=nid2[0],
                       balanced=world > 1)
        nd = len(doc_off) - 1
        cuts = sorted({0, nd} | {int(np.searchsorted(doc_off, T * k // S)) for k in range(1, S)})
        parts = []
        for a, b in zip(cuts, cuts[1:]):
            o = torch.from_numpy((doc_off[a:b + 1] - doc_off[a]).astype(np.int64)).pin_memory()
            parts.append((text_h[int(doc_off[a]):int(doc_off[b])], o))

        def e2e_step():
            ixe.reset()
            for t, o in parts:
                ixe.add_stream(t, o)
            ixe.finalize()

        e2e_step()
        out_bytes = ixe.serialized_size()
        out_h = torch.empty(out_bytes, dtype=torch.uint8, pin_memory=True)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        f0 = torch.cuda.Event(enable_timing=True)
        f1 = torch.cuda.Event(enable_timing=True)
        f0.record()
        for _ in range(args.e2e_steps):
            e2e_step()
            ixe.serialize_into(out_h.data_ptr(), out_bytes)
        f1.record()
        torch.cuda.synchronize()
        ems = f0.elapsed_time(f1) / args.e2e_steps
        if world > 1:
            t = torch.tensor([ems], device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ems = float(t.item())
        ixe.close()
        return {"value": total_bytes / (ems / 1e3) / 1e6, "unit": "MB/s", "ms_per_step": ems,
                "h2d_bytes_per_step": T + 8 * (nd + len(parts)), "d2h_bytes_per_step": out_bytes,
                "host_chunks": len(parts),
                "what": ("index_add_stream(pinned host text + doc_off%s) + index_finalize + index_serialize (%s) to "
                         "pinned host" % (f", {len(parts)} chunks, WJ_FLAG_HOST_PIPELINE" if len(parts) > 1 else "",
                                          "WJINV002 d-gap + vbyte postings" if vbyte else "WJINV001"))}

    e2e = e2e_vbyte = None
    if args.e2e_steps > 0:
        e2e = e2e_leg(args.vbyte)
        if not args.vbyte:  # the compressed output format: less than half the D2H bytes
            e2e_vbyte = e2e_leg(True)

    steady = None
    if args.steady_chunks > 0 and world == 1 and not force_dist:
        steady = steady_state(wj, ixp, args, local)  # (profiled context: its per-phase / per-kernel ms)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(text, doc_off)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "MB/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic (gen/wjgen.cpp seeded generator)",
            "config": {"workload": WORKLOAD.get(args.config, str(args.config)), "bytes_per_gpu": T,
                       "docs_per_gpu": len(doc_off) - 1, "tokens_per_gpu": N, "terms_per_gpu": V,
                       "postings_per_gpu": P, "stream_elems_per_gpu": E, "l2": "no flush: 1 GiB input per step > 126 MB L2",
                       "postings_format": "vbyte d-gaps (WJINV002)" if args.vbyte else "u32 docid + u32 tf (WJINV001)",
                       "parallelism": "single GPU" if world == 1 else
                       f"{world} ranks: document ranges, trie collections bin-packed by sampled load (P:212), NCCL all-to-all-v"},
            "exchange": exchange,
            "mib_per_s": total_bytes / (ms / 1e3) / 2**20,
            "tokens_per_s": N * world / (ms / 1e3),
            "roofline": {"bound": "hbm", "scope": "whole step (SURVEY 8(d) compulsory bytes)", "achieved": step_gbs,
                         "peak": peak * world, "unit": "GB/s", "frac": step_gbs / (peak * world),
                         "frac_of_nominal_8tbs": step_gbs / (8000.0 * world), "bytes_min": b_min,
                         "traffic": traffic, "traffic_ratio": (traffic / b_min) if traffic else None,
                         "peak_source": peak_src,
                         "def": ("B_min = T + (vbyte code bytes if --vbyte else 8P) + sum(len+28) over terms per step "
                                 "(SURVEY 8(d)) / step time / measured HBM copy bandwidth; traffic = ncu DRAM "
                                 "read+write bytes summed over one pass's launches (profiles/ncu_traffic.json)")},
            "kernel_efficiency": {"kernel": dom, "achieved": achieved, "peak": peak, "unit": "GB/s",
                                  "frac": achieved / peak, "algorithmic_bytes_per_launch": bytes_per_launch,
                                  "ms_per_launch": per_launch_ms, "launches_per_step": kcnt[dom] / args.steps,
                                  "def": "implementation bytes of DESIGN.md section 7 (design evidence, not the headline)"},
            "cpu_baseline": cpu,
            "e2e": e2e,
            "e2e_vbyte": e2e_vbyte,
            "steady_state": steady,
            "gpu_launches": int(round(launches * args.steps)),
            "gpu_launches_per_step": launches,
            "host_syncs_per_step": (s1["host_syncs"] - s0["host_syncs"]) / args.steps,
            "clocks": clk,
            "phases_ms_per_step": phases,
            "kernels": kernels,
            "breakdown": ("phases_ms_per_step / kernels / steady_state from a second context with CUDA-event "
                          "instrumentation, %d steps; the timed context runs without it" % prof_steps),
            "paper_context": "262.76 MB/s end-to-end on ClueWeb09 (2x X5560 + 2x C1060, Table VI); not this workload",
        }
        print_json(line)
    ixp.close()
    ix.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
