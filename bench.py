#!/usr/bin/env python
"""Benchmark of the Gallatin hot path on B200 (BASELINE.json metric:
"malloc+free ops/s per B200 (single/mixed size); vEB successor ops/s").

Workload at N=1: BASELINE configs[1], the single-size sweep (PAPER.md S6.5,
P:309-315) on a 16 GB heap: one STEP = for every slice size s in 16 B..4 KB,
reset the allocator, n_s = min(2^24, 8 GiB / s) threads each malloc(s)
(bulk kernel), then the same threads free.  value = (malloc + free ops) / time.
The line also carries the mixed-size cell (configs[2] shape, 2^22 threads on a
64 GB heap) and the vEB successor throughput (configs[0] tree, 2^24 queries).

Multi-GPU: one process per GPU (torchrun), independent per-GPU heaps ("replicas
only"); value = all ranks' ops / max-over-ranks time.

--impl reference times the CPU oracle (oracle/, O2) on a bounded sample of the
same workload (the reference arm of this tier: a deliberately slow program).
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
if os.environ.get("GALLATIN_PKG_ROOT"):            # same-box A/B of another build (tools/ab_build.sh)
    sys.path.insert(0, os.environ["GALLATIN_PKG_ROOT"])

import numpy as np  # noqa: E402

SEG = 1 << 24
HEAP_C2 = 16 << 30
HEAP_C3 = 64 << 30
SIZES = [16 << i for i in range(9)]


def cells_c2(scale: int = 1):
    """(size, threads) of the sweep: 2^20..2^24 threads, capped so that s*n <= 8 GiB
    (the feasible cells of SURVEY 8(d) C2); the largest feasible n per size."""
    return [(s, min(1 << 24, (8 << 30) // s) // scale) for s in SIZES]


# ------------------------------------------------------------------ clocks ---
class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled DURING the timed region."""
    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows: list[list[str]] = []
        self.proc = None
        self.thread = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "20"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
            return
        self.thread = threading.Thread(target=self._read, daemon=True)
        self.thread.start()

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self) -> dict:
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        if self.thread:
            self.thread.join(timeout=2)
        rows = [r for r in self.rows if len(r) >= 6 and r[0].replace(".", "").isdigit()]
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"], "samples": 0}
        sm = [float(r[0]) for r in rows]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[2 + i].lower().startswith("active")})
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": float(rows[0][1]), "reasons": reasons,
                "samples": len(rows)}


# ------------------------------------------------------------- distributed ---
def dist_setup(ngpus: int):
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != ngpus and world > 1:
        raise SystemExit(f"--gpus {ngpus} but WORLD_SIZE={world}")
    return rank, world, local


class Dist:
    """Process-group plumbing for independent per-GPU replicas: a barrier and
    max/sum of host scalars (no data-path collective exists)."""

    def __init__(self, rank, world, backend):
        self.rank, self.world = rank, world
        self.pg = None
        self.device = "cuda" if backend == "nccl" else "cpu"
        if world > 1:
            import torch.distributed as dist
            dist.init_process_group(backend)
            self.pg = dist

    def barrier(self):
        if self.pg:
            self.pg.barrier()

    def max(self, x: float) -> float:
        if not self.pg:
            return x
        import torch
        t = torch.tensor([x], dtype=torch.float64, device=self.device)
        self.pg.all_reduce(t, op=self.pg.ReduceOp.MAX)
        return float(t.item())

    def sum(self, x: float) -> float:
        if not self.pg:
            return x
        import torch
        t = torch.tensor([x], dtype=torch.float64, device=self.device)
        self.pg.all_reduce(t, op=self.pg.ReduceOp.SUM)
        return float(t.item())

    def close(self):
        if self.pg:
            self.pg.destroy_process_group()


def aggregate(d: "Dist", ops_local: float, ms_local: float) -> tuple[float, float, float]:
    """Whole-job throughput of independent replicas: every rank's ops over the
    slowest rank's device time.  Returns (value ops/s, max ms, total ops)."""
    ms = d.max(ms_local)
    total = d.sum(ops_local)
    return total / (ms / 1e3), ms, total


def peaks_file() -> dict:
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


# ------------------------------------------------------------- our arm -------
def run_ours(args, rank, world, local):
    import torch
    import paper_conf_ppopp_mccoyp24_b200 as G

    torch.cuda.set_device(local)
    d = Dist(rank, world, "nccl")
    stream = torch.cuda.current_stream()
    cells = cells_c2(args.scale)

    G.gallatin_init(HEAP_C2)
    size_t = [torch.full((n,), s, dtype=torch.int64, device="cuda") for s, n in cells]
    nmax = max(n for _, n in cells)
    ptrs = torch.empty(nmax, dtype=torch.int64, device="cuda")
    ops_per_step = sum(2 * n for _, n in cells)

    ev = {"m0": [], "m1": [], "f0": [], "f1": []}

    def step(record: bool, st_=None):
        # calls go to the current stream (the capture stream under a graph,
        # st_); graph-captured timing events are recorded as external nodes
        cur = torch.cuda.current_stream()
        ext = st_ is not None
        for (s, n), st in zip(cells, size_t):
            p = ptrs[:n]
            G.gallatin_reset()
            if record:
                e = torch.cuda.Event(enable_timing=True, external=ext); e.record(cur); ev["m0"].append(e)
            G.gallatin_malloc(st, p)
            if record:                                   # one event node ends the malloc and starts the free
                e = torch.cuda.Event(enable_timing=True, external=ext); e.record(cur)
                ev["m1"].append(e)
                ev["f0"].append(e)
            G.gallatin_free(p)
            if record:
                e = torch.cuda.Event(enable_timing=True, external=ext); e.record(cur); ev["f1"].append(e)

    # correctness gate on the bench's own launch configuration (untimed): the
    # first cell's pointers stamp/verify clean and the heap drains to pristine
    for w in range(max(args.warmup, 3)):
        step(False)
    torch.cuda.synchronize()
    (s0, n0), st0 = cells[0], size_t[0]
    G.gallatin_reset()
    G.gallatin_malloc(st0, ptrs[:n0])
    G.gallatin_stamp(ptrs[:n0], st0)
    bad = G.gallatin_verify(ptrs[:n0], st0)
    G.gallatin_free(ptrs[:n0])
    torch.cuda.synchronize()
    if bad:
        raise SystemExit(f"stamp-verify failed: {bad} words")

    # the K timed steps as one CUDA graph (same launches, no host launch gaps
    # between the step's 27 kernels), replayed once untimed to upload it
    # Two graphs of the same K steps: `graph` (no timing nodes) is the timed
    # region of `value`; `graph_ev` adds an event node around every malloc and
    # free call and is replayed afterwards for the per-kernel times (event
    # nodes sit on the critical path between kernels: ms_per_step_with_events)
    graph = graph_ev = None
    if args.graph:
        graph = torch.cuda.CUDAGraph()
        graph_ev = torch.cuda.CUDAGraph()
        cap = torch.cuda.Stream()
        cap.wait_stream(stream)
        with torch.cuda.graph(graph, stream=cap):
            for _ in range(args.steps):
                step(False, cap)
        with torch.cuda.graph(graph_ev, stream=cap):
            for _ in range(args.steps):
                step(True, cap)
        graph.replay()
        graph_ev.replay()
        torch.cuda.synchronize()
    clk = ClockSampler(local)
    d.barrier()
    torch.cuda.synchronize()
    clk.start()
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    t0.record(stream)
    if graph is not None:
        graph.replay()
    else:
        for _ in range(args.steps):
            step(True)
    t1.record(stream)
    torch.cuda.synchronize()
    clocks = clk.stop()
    d.barrier()
    ms_local = t0.elapsed_time(t1)
    value, ms, total_ops = aggregate(d, ops_per_step * args.steps, ms_local)
    ms_ev = None
    if graph_ev is not None:                       # the per-kernel event times
        t0.record(stream)
        graph_ev.replay()
        t1.record(stream)
        torch.cuda.synchronize()
        ms_ev = t0.elapsed_time(t1) / args.steps

    # per-kernel times (the roofline's dominant kernel)
    m_ms = [a.elapsed_time(b) for a, b in zip(ev["m0"], ev["m1"])]
    f_ms = [a.elapsed_time(b) for a, b in zip(ev["f0"], ev["f1"])]
    nsum = sum(n for _, n in cells) * args.steps
    malloc_ops_s = nsum / (sum(m_ms) / 1e3)
    free_ops_s = nsum / (sum(f_ms) / 1e3)
    per_cell = {}
    for i, (s, n) in enumerate(cells):
        mi, fi = m_ms[i::len(cells)], f_ms[i::len(cells)]
        mm, fm = statistics.median(mi), statistics.median(fi)
        per_cell[str(s)] = {"n": n, "malloc_ms": round(mm, 4), "free_ms": round(fm, 4),
                            "malloc_ms_p10_p90": [round(x, 4) for x in pctl(mi)],
                            "free_ms_p10_p90": [round(x, 4) for x in pctl(fi)],
                            "malloc_ops_s": n / mm * 1e3, "free_ops_s": n / fm * 1e3}

    # the replayed steps left a correct allocator: no bad free was counted,
    # and draining gives back every segment (the pristine state, by stats)
    G.gallatin_drain()
    st = G.gallatin_stats()
    if st["errors"] or st["free_segments"] != st["num_segments"] or any(st["tree_segments"]) or st["large_segments"]:
        raise SystemExit(f"allocator state after the timed steps is not pristine: {st}")
    rmw = count_rmws(G, torch, cells, size_t, ptrs)
    dominant = "malloc" if sum(m_ms) >= sum(f_ms) else "free"
    bytes_per_op = 16 if dominant == "malloc" else 8
    kern_ms = sum(m_ms) if dominant == "malloc" else sum(f_ms)
    achieved = nsum * bytes_per_op / (kern_ms / 1e3) / 1e9
    pk = peaks_file()
    hbm_peak = pk.get("hbm_gbs")
    peak_src = "MEASURED_PEAKS.json hbm_gbs"
    if not hbm_peak:
        hbm_peak, peak_src = 6650.0, "B200_PROFILING.md fallback"
    # traffic: DRAM bytes per launch of the dominant kernel on a 2^24-thread
    # cell, from the committed ncu --set full capture (profiles/traffic.json);
    # compare with the algorithmic bytes of that launch (16 or 8 B x 2^24)
    traffic = None
    tf = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tf):
        try:
            traffic = json.load(open(tf))["per_cell"][f"k_bulk_{dominant}"]["16"]
        except Exception:
            traffic = None

    extras = {}
    if not args.no_extras:
        extras = run_extras(args, G, torch, stream)

    # e2e through the C-ABI with HOST buffers (pinned), copies inside the timed region
    e2e = run_e2e(args, G, torch, cells)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = cpu_baseline(args)

    G.gallatin_destroy()
    if rank == 0:
        line = {
            "metric": "malloc+free ops/s per B200 (single-size sweep 16 B-4 KB)",
            "value": value, "unit": "ops/s", "n_gpus": world, "steps": args.steps, "warmup": max(args.warmup, 3),
            "ms_per_step": ms / args.steps, "ms_per_step_with_events": ms_ev,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "u64", "data": "synthetic",
            "config": {"launch": ("one CUDA graph of the K timed steps (per-kernel times from a second graph "
                                  "with event nodes around each call)") if args.graph else "eager",
                       "workload": "BASELINE configs[1]: single-size sweep 16 B-4 KB, n_s=min(2^24, 8GiB/s) threads, "
                                   "16 GiB heap, reset+malloc+free per size" + (f" (1/{args.scale} scale)" if args.scale > 1 else ""),
                       "heap_bytes": HEAP_C2, "cells": [[s, n] for s, n in cells],
                       "ops_per_step": ops_per_step, "parallelism": f"replicas x{world}",
                       "l2": "no flush: each step reads %.2f GiB of sizes + writes/reads the pointer array (> 126 MB L2)" % (
                           sum(8 * n for _, n in cells) / 2 ** 30)},
            "malloc_ops_s": malloc_ops_s, "free_ops_s": free_ops_s, "per_size": per_cell, "rmw_counts": rmw,
            "roofline": {"bound": "hbm", "kernel": "k_bulk_malloc_cta<8,10,128>" if dominant == "malloc" else "k_bulk_free_w<4,64,32>", "achieved": achieved, "peak": hbm_peak,
                         "unit": "GB/s", "frac": achieved / hbm_peak, "traffic": traffic,
                         "traffic_algorithmic": bytes_per_op * (1 << 24),
                         "traffic_note": "DRAM bytes of one 2^24-thread launch (16 B cell, profiles/r1_kernels.md)",
                         "algorithmic_bytes_per_op": bytes_per_op, "peak_source": peak_src},
            "clocks": clocks,
            "e2e": e2e,
            "gpu_launches": 36 * args.steps,             # per cell: k_reset, k_bulk_malloc_cta, k_big, k_bulk_free_w
            "cpu_baseline": cpu,
        }
        line.update(extras)
        line["fractions"] = fractions(line, hbm_peak)
        print(json.dumps(line))
    d.close()


def pctl(xs):
    """(p10, p90) of a sample."""
    a = np.sort(np.asarray(xs, dtype=float))
    return float(np.percentile(a, 10)), float(np.percentile(a, 90))


def count_rmws(G, torch, cells, size_t, ptrs) -> dict:
    """Per cell, the L2 RMWs the bulk kernels issue at minimum (SURVEY 8(d)
    "Algorithmic work per unit"): malloc = one slot RMW per class per
    1024-request CTA tile (single size: ceil(n / 1024)); free = one counter RMW
    per (warp, block) team, counted from the pointers one malloc returns (lane
    l of warp w frees ptrs[128 w + 32 k + l]: teams per 32-pointer row)."""
    base = G.gallatin_stats()["heap_base"]
    out = {}
    for (s, n), st in zip(cells, size_t):
        G.gallatin_reset()
        p = ptrs[:n]
        G.gallatin_malloc(st, p)
        c = max(0, (s - 1).bit_length() - 4)
        rows = (n + 31) // 32
        g = torch.full((rows * 32,), -1, dtype=torch.int64, device="cuda")
        g[:n] = (p - base) >> (16 + c)
        g = torch.sort(g.view(rows, 32), dim=1).values
        teams = int(((g[:, 1:] != g[:, :-1]).sum() + rows).item())
        G.gallatin_free(p)
        out[str(s)] = {"malloc_slot_rmws": (n + 1023) // 1024, "free_team_rmws": teams, "nslot": G.gallatin_stats()["nslot"][c]}
    torch.cuda.synchronize()
    G.gallatin_reset()
    return out


def fractions(line: dict, hbm_peak: float) -> dict:
    """Roofline fractions of every config (BASELINE north_star: "give each as
    absolute ops/s and as a fraction of the atomic/HBM roofline").  Peaks: the
    same-session probes (PK1-PK7) and MEASURED_PEAKS hbm_gbs."""
    pk = line.get("probes")
    fr = {}
    per = line["per_size"]
    rmw = line["rmw_counts"]
    tm = sum(v["malloc_ms"] for v in per.values())
    tf = sum(v["free_ms"] for v in per.values())
    n_all = sum(v["n"] for v in per.values())
    c2 = {"frac_hbm_malloc": n_all * 16 / (tm / 1e3) / 1e9 / hbm_peak,
          "frac_hbm_free": n_all * 8 / (tf / 1e3) / 1e9 / hbm_peak}
    if pk:
        a_dist32 = pk["atom_distinct"]["u32_random"]
        per_cell = {}
        for sz, v in per.items():
            r = rmw[sz]
            a_hot = pk["atom_hot"].get(str(r["nslot"])) or pk["atom_hot"]["148"]
            per_cell[sz] = {
                "frac_atom_malloc": (r["malloc_slot_rmws"] / (v["malloc_ms"] / 1e3)) / a_hot,
                "frac_atom_free": (r["free_team_rmws"] / (v["free_ms"] / 1e3)) / a_dist32,
                "frac_bump": v["malloc_ops_s"] / pk["bump_cta_16B"],
                "frac_hbm_malloc": v["n"] * 16 / (v["malloc_ms"] / 1e3) / 1e9 / hbm_peak,
                "frac_hbm_free": v["n"] * 8 / (v["free_ms"] / 1e3) / 1e9 / hbm_peak}
        c2["frac_atom_malloc"] = sum(rmw[k]["malloc_slot_rmws"] for k in per) / (tm / 1e3) / pk["atom_hot"]["148"]
        c2["frac_atom_free"] = sum(rmw[k]["free_team_rmws"] for k in per) / (tf / 1e3) / a_dist32
        c2["frac_bump"] = line["malloc_ops_s"] / pk["bump_cta_16B"]
        c2["per_size"] = per_cell
        c2["peaks_used"] = {"A_hot(NSLOT)": "probes.atom_hot[NSLOT(c)]", "A_dist": "probes.atom_distinct.u32_random",
                            "bump": "probes.bump_cta_16B (PK5b: 1 RMW per 512-request tile + 16 B I/O)"}
    fr["C2"] = c2
    if "veb" in line and pk:
        v = line["veb"]
        fr["C1_veb"] = {
            "successor_frac_hbm": v["successor_ops_s"] * 16 / 1e9 / hbm_peak,
            "successor_frac_l2_load": v["successor_ops_s"] / pk["load_random_8B_L2_16MB"],
            "insert_frac_atom": v["insert_ops_s"] / pk["atom_distinct"]["u64_random"],
            "delete_frac_atom": v["delete_ops_s"] / pk["atom_distinct"]["u64_random"],
            "note": "successor: >= 1 dependent 8 B tree load per query (L2 random-load rate, PK6) + 16 B HBM; "
                    "insert/delete: >= 1 distinct-address RMW per key (PK1 u64)"}
        big = {}
        for k, b in v.get("large_universes", {}).items():
            big[k] = {"successor_frac_hbm": b["successor_ops_s"] * 16 / 1e9 / hbm_peak,
                      "successor_frac_l2_load": b["successor_ops_s"] / pk["load_random_8B_L2_16MB"],
                      "successor_frac_hbm_random_load": b["successor_ops_s"] / pk["load_random_8B_HBM_4GB"],
                      "insert_frac_atom": b["insert_ops_s"] / pk["atom_distinct"]["u64_random"]}
        fr["C1_veb"]["large_universes"] = big
    if "mixed" in line:
        m = line["mixed"]
        fr["C3"] = {"frac_hbm_malloc": m["malloc_ops_s"] * 16 / 1e9 / hbm_peak,
                    "frac_hbm_free": m["free_ops_s"] * 8 / 1e9 / hbm_peak}
        if pk:
            fr["C3"]["frac_bump"] = m["malloc_ops_s"] / pk["bump_cta_16B"]
    if "thread_scaling" in line:
        fr["C4"] = {n: {"frac_hbm_malloc": v["malloc_ops_s"] * 16 / 1e9 / hbm_peak,
                        "frac_hbm_free": v["free_ops_s"] * 8 / 1e9 / hbm_peak}
                    for n, v in line["thread_scaling"]["points"].items()}
    if "graph" in line:
        bpe = {"init": 12, "bulk_insert": 12, "bulk_delete": 8, "expansion": 4, "edge_insert": 12, "edge_delete": 8}
        fr["C5"] = {k: {"frac_hbm_min": v["edges_per_s"] * bpe[k] / 1e9 / hbm_peak, "bytes_per_edge_min": bpe[k]}
                    for k, v in line["graph"]["phases"].items() if k in bpe}
        fr["C5"]["note"] = "lower-bound bytes per edge (8 B src+dst read, 4 B list write; deletes read 8 B); " \
                           "list copies on grow/shrink not counted"
    return fr


def run_extras(args, G, torch, stream):
    """Mixed-size cell, vEB successor throughput, peak probes (not part of `value`)."""
    import workload_gen as wg
    out = {}
    # --- vEB successor (configs[0] tree, 2^24 queries) ---
    w = wg.veb_workload(20, 1 << 16)
    v = G.Veb(20)
    keys = torch.from_numpy(w["insert"].view(np.int64)).cuda()
    nq = (1 << 24) // args.scale
    q = torch.from_numpy(wg.uniform_below(wg.cell_seed(1, 7), nq, 1 << 20).view(np.int64)).cuda()
    res = torch.empty_like(q)
    v.insert(keys, want_out=False)
    for _ in range(3):
        v.successor(q, res)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    reps = 20
    e0.record(stream)
    for _ in range(reps):
        v.successor(q, res)
    e1.record(stream)
    torch.cuda.synchronize()
    succ_ms = e0.elapsed_time(e1) / reps
    # insert/delete throughput on the same universe: R rounds of (clear,
    # insert the 2^16 keys, delete the 2^16 delete keys), events between the
    # back-to-back launches, median per launch
    dk = torch.from_numpy(w["delete"].view(np.int64)).cuda()
    ins_l, del_l = [], []
    for r in range(12):
        v.clear()
        ea, eb, ec = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        ea.record(stream)
        v.insert(keys, want_out=False)
        eb.record(stream)
        v.delete(dk, want_out=False)
        ec.record(stream)
        torch.cuda.synchronize()
        if r >= 2:
            ins_l.append(ea.elapsed_time(eb))
            del_l.append(eb.elapsed_time(ec))
    ins_ms_eager, del_ms_eager = statistics.median(ins_l), statistics.median(del_l)

    def vbody(mark):
        v.clear()
        mark()
        v.insert(keys, want_out=False)
        mark()
        v.delete(dk, want_out=False)
        mark()
    il, dl = graph_phases(torch, vbody, 10)
    ins_ms, del_ms = statistics.median(il), statistics.median(dl)
    v.close()
    out["veb"] = {"successor_ops_s": nq / succ_ms * 1e3, "successor_queries": nq, "successor_ms": succ_ms,
                  "insert_ops_s": len(w["insert"]) / ins_ms * 1e3, "delete_ops_s": len(w["delete"]) / del_ms * 1e3,
                  "insert_ms": ins_ms, "delete_ms": del_ms, "insert_ms_eager": ins_ms_eager,
                  "delete_ms_eager": del_ms_eager,
                  "insert_delete_timing": "graph-replayed rounds (device time); *_eager: events around eager launches",
                  "universe": "2^20", "keys": len(w["insert"]),
                  "successor_hbm_gbs": nq * 16 / succ_ms / 1e6}

    # --- successor on larger universes: 2^24 keys, 2^24 uniform queries ---
    big = {}
    for k in (24, 28, 32):
        vb = G.Veb(k)
        nk = min(1 << 24, (1 << k) >> 2)
        bk = torch.from_numpy(wg.distinct_below(wg.cell_seed(1, 400 + k), nk, 1 << k).view(np.int64)).cuda()
        bq = torch.from_numpy(wg.uniform_below(wg.cell_seed(1, 500 + k), nq, 1 << k).view(np.int64)).cuda()
        br = torch.empty_like(bq)
        vb.insert(bk, want_out=False)                 # warm-up round (then cleared)
        vb.clear()
        e0.record(stream)
        vb.insert(bk, want_out=False)
        e1.record(stream)
        torch.cuda.synchronize()
        bins = e0.elapsed_time(e1)
        for _ in range(3):
            vb.successor(bq, br)
        e0.record(stream)
        for _ in range(reps):
            vb.successor(bq, br)
        e1.record(stream)
        torch.cuda.synchronize()
        bms = e0.elapsed_time(e1) / reps
        big[f"2^{k}"] = {"keys": nk, "queries": nq, "insert_ops_s": nk / bins * 1e3, "successor_ops_s": nq / bms * 1e3,
                         "successor_ms": bms, "leaf_bytes": (1 << k) // 8}
        vb.close()
        del bk, bq, br
    out["veb"]["large_universes"] = big

    # --- mixed-size cell (configs[2] shape) on its own 64 GiB heap ---
    G.gallatin_destroy()
    G.gallatin_init(HEAP_C3)
    n = (1 << 22) // args.scale
    sizes = torch.from_numpy(wg.mixed_sizes(n).view(np.int64)).cuda()
    p = torch.empty_like(sizes)
    mm, fm = [], []
    for it in range(8):
        G.gallatin_reset()
        a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        a.record(stream)
        G.gallatin_malloc(sizes, p)
        b.record(stream)
        G.gallatin_free(p)
        c.record(stream)
        torch.cuda.synchronize()
        if it >= 3:
            mm.append(a.elapsed_time(b))
            fm.append(b.elapsed_time(c))
    me, fe = statistics.median(mm), statistics.median(fm)
    m, f = malloc_free_graph(G, torch, sizes, p)
    out["mixed"] = {"threads": n, "malloc_ops_s": n / m * 1e3, "free_ops_s": n / f * 1e3,
                    "combined_ops_s": 2 * n / (m + f) * 1e3, "malloc_ms": m, "free_ms": f,
                    "malloc_ms_eager": me, "free_ms_eager": fe,
                    "timing": "medians of 7 reset+malloc+free rounds replayed as one CUDA graph; *_eager: events "
                              "around eager launches",
                    "workload": "BASELINE configs[2]: 16 B-4 KB powers of two + p=2^-12 large 1-64 MB, 64 GiB heap"}
    G.gallatin_destroy()
    G.gallatin_init(HEAP_C2)

    out["probes"] = run_probes(G)
    out["grid"] = run_grid(args, G, torch, stream)
    out["thread_scaling"] = run_scaling(args, G, torch, stream)
    out["graph"] = run_graph(args, G, torch, stream)
    out["paper_modes"] = run_paper_modes(args, G, torch)
    return out


def run_grid(args, G, torch, stream) -> dict:
    """BASELINE configs[1] as a full grid: every size 16 B..4 KB
    x n = 2^20..2^24 threads on the 16 GiB heap.  The 39 cells with s*n <= 8 GiB
    are timed (reset before every repetition; median and p10/p90 of 5
    rounds replayed as one CUDA graph, `graph_phases`);
    the 6 others are capacity runs (one call asking more than the heap holds:
    NULL count and time).  At the headline n of every size, warm rounds (no
    reset, after one untimed round) are timed beside the cold ones."""
    ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
    reps = 5
    cells, cap_runs, warm = {}, {}, {}
    for s in SIZES:
        for lg in range(20, 25):
            n = (1 << lg) // args.scale
            st = torch.full((n,), s, dtype=torch.int64, device="cuda")
            p = torch.empty_like(st)
            if s * (1 << lg) > (8 << 30):
                G.gallatin_reset()
                a, b = ev(), ev()
                a.record(stream)
                G.gallatin_malloc(st, p)
                b.record(stream)
                torch.cuda.synchronize()
                nulls = int((p == 0).sum().item())
                cap_runs[f"{s}x2^{lg}"] = {"n": n, "nulls": nulls, "granted": n - nulls, "malloc_ms": a.elapsed_time(b),
                                           "granted_bytes": (n - nulls) * s}
                G.gallatin_free(p)
                continue
            def cold(mark):
                G.gallatin_reset()
                mark()
                G.gallatin_malloc(st, p)
                mark()
                G.gallatin_free(p)
                mark()
            mm, fm = graph_phases(torch, cold, reps)
            m, f = statistics.median(mm), statistics.median(fm)
            cells[f"{s}x2^{lg}"] = {"n": n, "malloc_ms": round(m, 5), "free_ms": round(f, 5),
                                    "malloc_ms_p10_p90": [round(x, 5) for x in pctl(mm)],
                                    "free_ms_p10_p90": [round(x, 5) for x in pctl(fm)],
                                    "malloc_ops_s": n / m * 1e3, "free_ops_s": n / f * 1e3}
            if (1 << lg) == min(1 << 24, (8 << 30) // s):             # the headline cell: warm rounds
                G.gallatin_reset()
                G.gallatin_malloc(st, p)
                G.gallatin_free(p)                                   # the untimed first round

                def warm_round(mark):
                    mark()
                    G.gallatin_malloc(st, p)
                    mark()
                    G.gallatin_free(p)
                    mark()
                wm, wf = graph_phases(torch, warm_round, 2 * reps - 1)         # warm state drifts: 9 rounds
                warm[str(s)] = {"n": n, "cold_malloc_ms": round(m, 5), "warm_malloc_ms": round(statistics.median(wm), 5),
                                "cold_free_ms": round(f, 5), "warm_free_ms": round(statistics.median(wf), 5),
                                "warm_over_cold_malloc": statistics.median(wm) / m}
            del st, p
    G.gallatin_reset()
    return {"workload": "BASELINE configs[1] grid: 16 B..4 KB x 2^20..2^24 threads, 16 GiB heap", "reps": reps,
            "cells": cells, "capacity_runs": cap_runs, "warm_vs_cold": warm}


HOT_N = [1, 4, 9, 18, 37, 74, 148, 256, 302, 1024]       # slot-line counts


def run_probes(G) -> dict:
    """SURVEY 8(d) PK1-PK7 on persistent microkernels (probes.cu), same
    session as the configs.  Rates in operations per second."""
    def rate(kind, n, param):
        ms, ops = G.gallatin_probe(kind, n, param)
        return ops / ms * 1e3
    w16m = (16 << 20) // 8                       # a 16 MB L2-resident array of u64
    pk = {"atom_distinct": {
        "u64_random": rate(1, 1 << 27, w16m), "u32_random": rate(7, 1 << 27, 2 * w16m),
        "u64_coalesced": rate(8, 1 << 27, w16m), "u32_coalesced": rate(9, 1 << 27, 2 * w16m)}}
    pk["atom_hot"] = {str(n): rate(2, 1 << 24, n) for n in HOT_N}
    pk["red_hot"] = {str(n): rate(3, 1 << 24, n) for n in HOT_N}
    pk["cas_hot"] = {str(n): rate(10, 1 << 22, n) for n in HOT_N}
    pk["bump_warp_16B"] = rate(4, 1 << 24, 148)
    pk["bump_cta_16B"] = rate(11, 1 << 24, 148)
    pk["bump_cta_4KB_4slots"] = rate(11, 1 << 24, 4)
    pk["fence_acq_rel_per_warp"] = rate(5, 1 << 22, 1)
    pk["fence_sc_per_warp"] = rate(12, 1 << 22, 1)
    pk["load_random_8B_L2_16MB"] = rate(13, 1 << 27, w16m)
    pk["load_random_8B_HBM_4GB"] = rate(13, 1 << 26, (4 << 30) // 8)
    ms, ops = G.gallatin_probe(6, 1 << 24, 1 << 31)
    pk["hbm_copy_gbs"] = ops / ms / 1e6
    pk["units"] = "operations/s (atomics, loads, fences, bump requests); hbm_copy in GB/s"
    return pk


def run_paper_modes(args, G, torch):
    """PAPER.md S6's other modes (experiments.py): utilization on a 2 GB heap
    with batches of 100,000 (E8), fragmentation of 2^20 allocations
    (E7), warmed-up vs reset rounds at 2 KB (E6), the variance
    of 50 rounds (E5) and init time (E1)."""
    from paper_conf_ppopp_mccoyp24_b200 import experiments as X
    out = {}
    G.gallatin_destroy()
    util = {}
    for size in [4 << i for i in range(12)]:                    # 4 B .. 8 KB
        G.gallatin_init(2 << 30)
        r = X.utilization(size, batch=100_000 // args.scale)
        util[str(size)] = {"utilization": round(r["utilization"], 4), "successes": r["successes"],
                           "batches": r["batches"]}
        del r
        G.gallatin_destroy()
    out["utilization"] = {"heap_bytes": 2 << 30, "batch": 100_000 // args.scale, "per_size": util,
                          "note": "successes x size / heap; sizes < 16 B round up to 16 B slices, "
                                  "8 KB takes a 64 KB block (reading A-2)"}
    # fragmentation with the default knobs (runs of blocks per slot) and with
    # the paper's one-block buffer (run_max = run_init = 1, no format-ahead)
    out["fragmentation"] = {"n": (1 << 20) // args.scale}
    for name, knobs in (("default", {}), ("paper_policy", dict(run_max=1, run_init=1, format_ahead=2, prefetch=2, prefill=2))):
        G.gallatin_init(HEAP_C2, **knobs)
        frag = {}
        for size in SIZES:
            G.gallatin_reset()
            r = X.fragmentation(size, (1 << 20) // args.scale)
            frag[str(size)] = {"range_bytes": r["range_bytes"],
                               "range_over_requested": round(r["range_over_requested"], 4)}
            G.gallatin_free(r["ptrs"])
            del r
        out["fragmentation"][name] = frag
        G.gallatin_destroy()
    G.gallatin_init(HEAP_C2)
    out["warm_vs_cold_2KB"] = X.warm_vs_cold(2048, (1 << 20) // args.scale, rounds=20)
    out["variance_64B"] = X.variance(64, (1 << 20) // args.scale, rounds=50)
    G.gallatin_destroy()
    out["init"] = X.init_time(HEAP_C2, reps=3)
    G.gallatin_init(HEAP_C2)
    return out


def graph_phases(torch, body, reps: int):
    """Device time of each phase of body(mark), run `reps` times back to back as
    ONE CUDA graph (no host launch gaps inside the timed region; the timing
    events are graph nodes), replayed once to upload and once timed.  Phase i
    runs from the i-th to the (i+1)-th mark() of a rep; returns
    [[ms of phase i in rep r for r] for i]."""
    marks = []

    def mark():
        e = torch.cuda.Event(enable_timing=True, external=True)
        e.record(torch.cuda.current_stream())
        marks.append(e)

    g = torch.cuda.CUDAGraph()
    cap = torch.cuda.Stream()
    cap.wait_stream(torch.cuda.current_stream())
    with torch.cuda.graph(g, stream=cap):
        for _ in range(reps):
            body(mark)
    g.replay()
    torch.cuda.synchronize()
    g.replay()
    torch.cuda.synchronize()
    per = len(marks) // reps
    res = [[marks[r * per + i].elapsed_time(marks[r * per + i + 1]) for r in range(reps)] for i in range(per - 1)]
    del g
    return res


def malloc_free_graph(G, torch, st, p, reps: int = 7):
    """(malloc ms, free ms) medians of reset + malloc + free, graph-timed."""
    def body(mark):
        G.gallatin_reset()
        mark()
        G.gallatin_malloc(st, p)
        mark()
        G.gallatin_free(p)
        mark()
    mm, fm = graph_phases(torch, body, reps)
    return statistics.median(mm), statistics.median(fm)


def run_scaling(args, G, torch, stream):
    """BASELINE configs[3]: 64 B mallocs then frees at 2^10 .. 2^26 threads on the
    16 GiB heap (reset before each run); median of 5 runs per point."""
    pts = {}
    for lg in range(10, 27, 2):
        n = (1 << lg) // args.scale if (1 << lg) // args.scale >= 1024 else 1 << lg
        st = torch.full((n,), 64, dtype=torch.int64, device="cuda")
        p = torch.empty_like(st)
        mm, fm = [], []
        for it in range(7):
            G.gallatin_reset()
            a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            a.record(stream)
            G.gallatin_malloc(st, p)
            b.record(stream)
            G.gallatin_free(p)
            c.record(stream)
            torch.cuda.synchronize()
            if it >= 2:
                mm.append(a.elapsed_time(b))
                fm.append(b.elapsed_time(c))
        me, fe = statistics.median(mm), statistics.median(fm)
        m, f = malloc_free_graph(G, torch, st, p)
        pts[str(n)] = {"malloc_ms": round(m, 5), "free_ms": round(f, 5), "malloc_ops_s": n / m * 1e3,
                       "free_ops_s": n / f * 1e3, "malloc_ms_eager": round(me, 5), "free_ms_eager": round(fe, 5)}
        del st, p
    # the paper's other scaling sizes (16, 512, 8192 B) up to its 2^20 threads
    paper = {}
    for size in (16, 512, 8192):
        pp = {}
        for lg in range(10, 21, 2):
            n = max(1024, (1 << lg) // args.scale)
            if size == 8192 and n * 65536 > HEAP_C2 // 2:
                continue                        # 8 KB takes a 64 KB block (A-2): > half the heap
            st = torch.full((n,), size, dtype=torch.int64, device="cuda")
            p = torch.empty_like(st)
            mm, fm = [], []
            for it in range(7):
                G.gallatin_reset()
                a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
                a.record(stream)
                G.gallatin_malloc(st, p)
                b.record(stream)
                G.gallatin_free(p)
                c.record(stream)
                torch.cuda.synchronize()
                if it >= 2:
                    mm.append(a.elapsed_time(b))
                    fm.append(b.elapsed_time(c))
            me, fe = statistics.median(mm), statistics.median(fm)
            m, f = malloc_free_graph(G, torch, st, p)
            pp[str(n)] = {"malloc_ms": round(m, 5), "free_ms": round(f, 5), "malloc_ops_s": n / m * 1e3,
                          "free_ops_s": n / f * 1e3, "malloc_ms_eager": round(me, 5), "free_ms_eager": round(fe, 5)}
        paper[str(size)] = pp
    return {"workload": "BASELINE configs[3]: 64 B, 2^10..2^26 threads (every 4th power), 16 GiB heap, "
                        "independent per-GPU heap under torchrun",
            "timing": "malloc_ms/free_ms: medians of 7 reset+malloc+free rounds replayed as one CUDA graph "
                      "(device time, no host launch gap); *_eager: the same calls with events around eager "
                      "launches (host ctypes launch latency included)",
            "points": pts,
            "paper_sizes": {"workload": "P:329 sizes 16/512/8192 B at 2^10..2^20 threads (every 2nd power)",
                            "points": paper}}


def run_graph(args, G, torch, stream):
    """BASELINE configs[4]: R-MAT 2^24 vertices / 2^28 edges on a 16 GiB heap;
    adjacency lists kept by DEVICE-side malloc/free (include/gallatin_graph.h).
    Edges/s per phase and the allocator calls the kernels issued."""
    import workload_gen as wg
    scale = 24 - max(0, int(np.log2(args.scale)))
    n = 1 << (scale + 4)
    G.gallatin_destroy()
    G.gallatin_init(HEAP_C2)
    w = wg.graph_workload(scale, n, device="cuda", n_expand=1 << 16)
    torch.cuda.synchronize()
    g = G.Graph(w["V"])
    ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
    res = {}

    def timed(name, fn, edges):
        a, b = ev(), ev()
        a.record(stream)
        fn()
        b.record(stream)
        torch.cuda.synchronize()
        ms = a.elapsed_time(b)
        res[name] = {"ms": ms, "edges": edges, "edges_per_s": edges / ms * 1e3}

    s0, d0 = w["init"]
    timed("init", lambda: g.insert(s0, d0), s0.numel())
    timed("bulk_insert", lambda: [g.insert(s, d) for s, d in w["insert"]], sum(s.numel() for s, _ in w["insert"]))
    timed("bulk_delete", lambda: [g.delete(s, d) for s, d in w["delete"]], sum(s.numel() for s, _ in w["delete"]))
    size, _, _ = g.export()
    before = int(size.sum())
    timed("expansion", lambda: [g.expand(w["expand"]) for _ in range(w["rounds"])], 0)
    size, cap, _ = g.export()
    res["expansion"]["edges"] = int(size.sum()) - before
    res["expansion"]["edges_per_s"] = res["expansion"]["edges"] / res["expansion"]["ms"] * 1e3
    # P:355's non-bulk variants: one thread per edge under a vertex lock, on
    # 2^22 edges of the stream (re-inserted, then deleted one at a time)
    ne = min(1 << 22, w["insert"][0][0].numel())
    es, ed = w["insert"][0][0][:ne].contiguous(), w["insert"][0][1][:ne].contiguous()
    timed("edge_insert", lambda: g.insert_edges(es, ed), ne)
    timed("edge_delete", lambda: g.delete_edges(es, ed), ne)
    ctr = g.counters()
    total_ms = sum(v["ms"] for v in res.values())
    g.destroy()
    G.gallatin_drain()
    st = G.gallatin_stats()
    G.gallatin_destroy()
    G.gallatin_init(HEAP_C2)
    return {"workload": f"BASELINE configs[4]: R-MAT 2^{scale} vertices / 2^{scale + 4} edges, (a,b,c,d)="
                        "(0.57,0.19,0.19,0.05), 8 insert + 8 delete batches, 2^16-vertex x 8-round expansion, "
                        "2^22 single-edge inserts + deletes, 16 GiB heap",
            "phases": res, "device_mallocs": ctr["mallocs"], "device_frees": ctr["frees"],
            "failed_mallocs": ctr["failed"], "allocator_ops_per_s": (ctr["mallocs"] + ctr["frees"]) / total_ms * 1e3,
            "pristine_after_teardown": st["free_segments"] == st["num_segments"]}


def run_e2e(args, G, torch, cells):
    """Same metric through gallatin_malloc_host / gallatin_free_host: the sizes are
    copied host->device, the pointers device->host (malloc) and host->device (free)."""
    host = []
    for s, n in cells:
        hs = torch.full((n,), s, dtype=torch.int64, pin_memory=True).numpy().view(np.uint64)
        hp = torch.empty(n, dtype=torch.int64, pin_memory=True).numpy().view(np.uint64)
        host.append((hs, hp))
    steps = max(1, min(args.steps, 5))
    for (hs, hp) in host:                                 # warm-up
        G.gallatin_reset()
        torch.cuda.synchronize()
        G.gallatin_malloc_host(hs, hp)
        G.gallatin_free_host(hp)
    torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(steps):
        for (hs, hp) in host:
            G.gallatin_reset()
            G.gallatin_malloc_host(hs, hp)
            G.gallatin_free_host(hp)
    torch.cuda.synchronize()
    dt = time.perf_counter() - t
    ops = sum(2 * n for _, n in cells) * steps
    return {"value": ops / dt, "unit": "ops/s", "h2d_bytes_per_step": sum(16 * n for _, n in cells),
            "d2h_bytes_per_step": sum(8 * n for _, n in cells), "steps": steps,
            "api": "gallatin_malloc_host/gallatin_free_host (pinned host arrays)"}


# ---------------------------------------------------------- CPU oracle ------
def cpu_sample(scale_div: int):
    """The bounded oracle sample: every cell at 1/scale_div of its threads."""
    return [(s, max(1, n // scale_div)) for s, n in cells_c2()]



def time_oracle(cells, steps: int):
    import oracle
    import workload_gen as wg
    os.sched_setaffinity(0, {sorted(os.sched_getaffinity(0))[0]})   # one host core
    sizes = [wg.single_sizes(s, n) for s, n in cells]
    total = 0.0
    ops = 0
    for _ in range(steps):
        for (s, n), sz in zip(cells, sizes):
            a = oracle.Allocator(HEAP_C2 // SEG)       # fresh = the paper's reset
            t = time.perf_counter()
            offs = a.malloc_batch(sz, keydiv=32)
            a.free_batch(offs)
            total += time.perf_counter() - t
            ops += 2 * n
            a.close()
    return ops, total


def host_cpu() -> dict:
    """The box's host CPU model and core count (north_star: "core count stated")."""
    model = "unknown"
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    return {"cpu_model": model, "nproc": os.cpu_count(), "affinity_cores": len(os.sched_getaffinity(0))}


def cpu_baseline(args):
    div = 8
    cells = cpu_sample(div)
    host = host_cpu()
    ops, sec = time_oracle(cells, 1)
    return {"value": ops / sec, "unit": "ops/s", "cores": 1, "kind": "oracle",
            "sample": f"O2-P (oracle/alloc_paper.c, the paper's policy) on every cell of the sweep at 1/{div} of "
                      f"its threads ({ops // 2} mallocs + frees), one pinned host core", "seconds": sec, **host}


def run_reference(args, rank, world):
    if rank != 0:                      # the reference arm runs on rank 0 only
        return
    div = 8 * args.scale
    cells = cpu_sample(div)
    host = host_cpu()
    steps = max(1, min(args.steps, 3))
    for _ in range(min(args.warmup, 1)):
        time_oracle(cells[:1], 1)
    ops, sec = time_oracle(cells, steps)
    value = ops / sec
    line = {
        "impl": "reference",
        "metric": "malloc+free ops/s per B200 (single-size sweep 16 B-4 KB)",
        "value": value, "unit": "ops/s", "n_gpus": world, "steps": steps, "warmup": args.warmup,
        "ms_per_step": sec / steps * 1e3, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": "u64", "data": "synthetic",
        "config": {"workload": "BASELINE configs[1]: single-size sweep 16 B-4 KB, 16 GiB heap; the CPU oracle "
                               f"runs each cell at 1/{div} of its threads", "cells": [[s, n] for s, n in cells]},
        "cpu_baseline": {"value": value, "unit": "ops/s", "cores": 1, "kind": "oracle",
                         "sample": f"O2-P on every cell at 1/{div} of its threads, {steps} step(s), one pinned host core",
                         **host},
        "e2e": {"value": value, "unit": "ops/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--scale", type=int, default=1, help="divide every thread count (debug only)")
    ap.add_argument("--no-extras", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-graph", dest="graph", action="store_false",
                    help="issue the timed steps eagerly instead of as one CUDA graph")
    args = ap.parse_args()
    rank, world, local = dist_setup(args.gpus)
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    run_ours(args, rank, world, local)


if __name__ == "__main__":
    main()
