#!/usr/bin/env python
"""bench.py — BFS GTEPS on the config-4 workload (Kronecker/R-MAT scale 24, edge factor 32,
permuted, direction-optimising), through the C ABI of libsygraph.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl sygraph|reference] [--config 4]

One *step* = one full BFS (all §8(a) rows: compaction, tiered push / pull advance, frontier
swap/clear, direction policy) from one of the 64 seeded roots.  `value` = Graph500 TEPS summed
over all ranks' steps / max-over-ranks device time (CUDA events, barrier + synchronize on both
sides).  N > 1: the 64 roots are independent problems sharded across ranks (weak scaling, no
data-path collective).  The graph (4 GB of col_idx) is larger than L2, so no flush is needed.
`e2e` = the same metric through graph_load_csr from pinned HOST buffers + run_bfs + level D2H per
step.  `--impl reference` times the oracle (queue BFS, one host core) on the same workload.
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

METRIC = "BFS GTEPS (Graph500 m_s / time), Kronecker scale-24 EF32, direction-optimising"
UNIT = "GTEPS"


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="sygraph", choices=["sygraph", "reference"])
    p.add_argument("--config", type=int, default=4)
    p.add_argument("--seed", type=int, default=1)
    p.add_argument("--direction", default="auto", choices=["auto", "push", "pull"])
    p.add_argument("--alpha", type=float, default=14.0)
    p.add_argument("--beta", type=float, default=24.0)
    p.add_argument("--heavy-degree", type=int, default=0, help="CTA/grid-tier degree threshold (0: library default)")
    p.add_argument("--scsr", type=int, default=0, help="segmented push advance: 0 auto, 1 off, 2 always")
    p.add_argument("--e2e-steps", type=int, default=3)
    p.add_argument("--dense-roots", type=int, default=3, help="push-only BFS roots for roofline_dense_push (0: skip)")
    p.add_argument("--cpu-seconds", type=float, default=15.0)
    p.add_argument("--no-cpu-baseline", action="store_true")
    return p.parse_args()


class ClockSampler:
    """SM clock + clock-event (throttle) reasons polled through NVML every ~2 ms during the timed
    region (the same counters `nvidia-smi --query-gpu=clocks.sm,clocks_event_reasons.*` reads;
    a 100 ms nvidia-smi loop cannot sample a ~10 ms region)."""
    REASONS = {"hw_slowdown": 0x8, "hw_thermal_slowdown": 0x40, "sw_thermal_slowdown": 0x20,
               "sw_power_cap": 0x4, "hw_power_brake_slowdown": 0x80}

    def __init__(self, index):
        self.index, self.samples, self.reason_bits, self.max_mhz = index, [], 0, None
        self._stop = threading.Event()

    def _poll(self):
        import pynvml as N
        while not self._stop.is_set():
            try:
                self.samples.append(N.nvmlDeviceGetClockInfo(self.h, N.NVML_CLOCK_SM))
                self.reason_bits |= N.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            except Exception:
                pass
            time.sleep(0.002)

    def __enter__(self):
        try:
            import pynvml as N
            N.nvmlInit()
            self.h = N.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = N.nvmlDeviceGetMaxClockInfo(self.h, N.NVML_CLOCK_SM)
            self._poll_once()
            self.t = threading.Thread(target=self._poll, daemon=True)
            self.t.start()
        except Exception:
            self.h = None
        return self

    def _poll_once(self):
        import pynvml as N
        self.samples.append(N.nvmlDeviceGetClockInfo(self.h, N.NVML_CLOCK_SM))
        self.reason_bits |= N.nvmlDeviceGetCurrentClocksEventReasons(self.h)

    def __exit__(self, *a):
        if getattr(self, "h", None) is not None:
            try:
                self._poll_once()
            except Exception:
                pass
            self._stop.set()
            self.t.join(timeout=1)

    def summary(self):
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None, "sm_max_mhz": self.max_mhz,
                "reasons": sorted(k for k, b in self.REASONS.items() if self.reason_bits & b),
                "samples": len(self.samples), "source": "nvml"}


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f).get("hbm_gbs", 6650.0), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


def committed_traffic():
    """Per-launch dram bytes of the dominant kernel from the committed ncu --set full summary."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            return json.load(f)
    except Exception:
        return None


def make_graph(cfg, seed, pinned):
    import gen
    import torch
    alloc = None
    if pinned:
        keep = {}

        def alloc(n, nnz):
            rp = torch.empty(n + 1, dtype=torch.int64, pin_memory=True)
            ci = torch.empty(max(nnz, 1), dtype=torch.int32, pin_memory=True)
            keep["rp"], keep["ci"] = rp, ci
            return rp.numpy(), ci.numpy()[:nnz]
    g = gen.make_config_graph(cfg, seed=seed, alloc=alloc)
    if pinned:
        g.meta["pinned"] = keep          # keep the pinned buffers alive with the graph
    return g


def m_s_of(level_u32_dev, deg_dev):
    """Graph500 m_s: undirected edges with an endpoint reached = sum of degrees of reached / 2."""
    import torch
    reached = level_u32_dev != -1
    return int(torch.sum(deg_dev[reached]).item()) // 2


def workload_config(args, g, world):
    """The `config` object both arms print (identical keys and values)."""
    return {"workload": f"config{args.config}: BFS from 64 seeded roots (stream 5), Kronecker/R-MAT scale 24 EF32, "
                        f"Graph500 A/B/C=.57/.19/.19, permuted, symmetric",
            "n": g.n, "nnz": g.nnz, "direction": args.direction, "step": "one full BFS from one root",
            "parallelism": f"roots sharded over {world} GPU(s)" if world > 1 else "1 GPU",
            "l2": "inputs larger than L2 (4 GB col_idx vs 126 MB L2)"}


def run_reference(args, rank):
    """Reference arm = the oracle (queue BFS, single host core) on the same workload."""
    if rank != 0:
        return 0
    import gen
    import oracle
    g = gen.make_config_graph(args.config, seed=args.seed)
    roots = gen.config_sources(args.config, g, seed=args.seed)
    deg = g.degrees()

    def step(i):
        s = int(roots[i % len(roots)])
        lv = oracle.bfs(g, s)
        return int(deg[lv != 0xFFFFFFFF].sum()) // 2

    for i in range(args.warmup):
        step(i)
    t0 = time.perf_counter()
    ms_total = 0
    for i in range(args.steps):
        ms_total += step(args.warmup + i)
    dt = time.perf_counter() - t0
    value = ms_total / dt / 1e9
    line = {"metric": METRIC, "value": value, "unit": UNIT, "impl": "reference", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": workload_config(args, g, args.gpus),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": f"{args.steps} timed queue-BFS roots (1 BFS per step)"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        os.environ.setdefault("OMP_NUM_THREADS", str(max(1, (os.cpu_count() or 8) // world)))
    if args.impl == "reference":
        return run_reference(args, rank)

    import torch
    import torch.distributed as dist
    import gen
    import paper_conf_icpp_carocc25_b200 as sg

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream()

    t_gen = time.perf_counter()
    g = make_graph(args.config, args.seed, pinned=True)
    t_gen = time.perf_counter() - t_gen
    roots_all = gen.config_sources(args.config, g, seed=args.seed)
    roots = roots_all[rank::world] if world <= len(roots_all) else roots_all[[rank % len(roots_all)]]
    rp_h = torch.from_numpy(g.row_ptr)
    ci_h = torch.from_numpy(g.col_idx)
    G = sg.graph_load_csr(rp_h, ci_h)                     # host -> device copy (not timed)
    deg = torch.diff(rp_h.to(dev))
    direction = {"auto": sg.SG_DIR_AUTO, "push": sg.SG_DIR_PUSH, "pull": sg.SG_DIR_PULL}[args.direction]
    o = sg.opts(stream=stream, direction=direction, alpha=args.alpha, beta=args.beta, heavy_degree=args.heavy_degree,
                 scsr=args.scsr)
    level = torch.empty(g.n, dtype=torch.int32, device=dev)

    # m_s per root (untimed; BFS results are deterministic per root)
    step_roots = [int(roots[(args.warmup + i) % len(roots)]) for i in range(args.steps)]
    ms_of = {}
    for s in sorted(set(step_roots) | {int(roots[i % len(roots)]) for i in range(max(args.e2e_steps, 1))}):
        sg.run_bfs(G, s, level, o)
        ms_of[s] = m_s_of(level, deg)
    for i in range(args.warmup):
        sg.run_bfs(G, int(roots[i % len(roots)]), level, o)

    # ---- timed region (device-resident inputs; each BFS is one CUDA graph launch) ----
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    stats = []
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    launches0 = sg.launch_count()
    with ClockSampler(local) as clk:
        ev0.record(stream)
        for s in step_roots:
            _, st = sg.run_bfs(G, s, level, o)
            stats.append(st.as_dict())
        ev1.record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    launches = sg.launch_count() - launches0
    ms = ev0.elapsed_time(ev1)

    # ---- per-kernel-class CUDA events: the same K roots, host-driven loop (a graph has no
    # per-launch events); gives the roofline of the dominant kernel and its share of a step ----
    sg.profile(G, True)
    p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    p0.record(stream)
    for s in step_roots:
        sg.run_bfs(G, s, level, o)
    p1.record(stream)
    torch.cuda.synchronize()
    prof = sg.profile_read(G)
    sg.profile(G, False)
    ms_prof = p0.elapsed_time(p1)
    edges = sum(ms_of[s] for s in step_roots)
    t_max = torch.tensor([ms], dtype=torch.float64, device=dev)
    e_sum = torch.tensor([edges], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t_max, op=dist.ReduceOp.MAX)
        dist.all_reduce(e_sum, op=dist.ReduceOp.SUM)
    ms_max = float(t_max.item())
    value = float(e_sum.item()) / (ms_max / 1e3) / 1e9

    # ---- roofline of the dominant kernel class ----
    dom = max(prof, key=lambda k: prof[k]["ms"])
    P = prof[dom]
    peak, peak_src = peaks()
    achieved = (P["bytes"] / P["launches"]) / (P["ms"] / P["launches"] / 1e3) / 1e9 if P["launches"] else 0.0
    tr = committed_traffic()
    roofline = {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "peak_source": peak_src,
                "traffic": (tr or {}).get(dom, {}).get("dram_bytes_per_launch") if tr else None,
                "bytes_per_launch": P["bytes"] / max(P["launches"], 1),
                "ms_per_launch": P["ms"] / max(P["launches"], 1),
                "share_of_step": P["ms"] / ms_prof if ms_prof else None,
                "measured_in": "CUDA events per launch on the launching stream, host-driven pass over the "
                               "timed region's K roots (ms_per_step %.3f there)" % (ms_prof / args.steps),
                "classes": {k: {"ms": v["ms"], "launches": v["launches"],
                                "GBps": (v["bytes"] / (v["ms"] / 1e3) / 1e9) if v["ms"] else 0.0}
                            for k, v in prof.items()}}

    # ---- the north star's HBM bar: the dense top-down advance (direction optimisation off) ----
    # push-only BFS over a few of the same roots, host-driven with per-class events; the dense
    # supersteps go through the destination-segmented sweep (class advance_sweep)
    dense = None
    if args.direction != "pull" and args.dense_roots > 0:
        od = sg.opts(stream=stream, direction=sg.SG_DIR_PUSH, heavy_degree=args.heavy_degree, scsr=args.scsr)
        d_roots = [int(roots[i % len(roots)]) for i in range(args.dense_roots)]
        sg.run_bfs(G, d_roots[0], level, od)   # untimed: builds the segment-major arc copy (lazy, R7)
        torch.cuda.synchronize()
        sg.profile(G, True)
        q0, q1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        q0.record(stream)
        for s in d_roots:
            sg.run_bfs(G, s, level, od)
        q1.record(stream)
        torch.cuda.synchronize()
        dprof = sg.profile_read(G)
        sg.profile(G, False)
        ms_d = q0.elapsed_time(q1)
        for s in d_roots:
            if s not in ms_of:
                sg.run_bfs(G, s, level, o)
                ms_of[s] = m_s_of(level, deg)
        D = dprof.get("advance_sweep", {"launches": 0})
        if D["launches"]:
            ach = (D["bytes"] / D["launches"]) / (D["ms"] / D["launches"] / 1e3) / 1e9
            dense = {"bound": "hbm", "kernel": "k_push_sweep (advance_sweep)", "achieved": ach, "peak": peak,
                     "unit": "GB/s", "frac": ach / peak, "peak_source": peak_src,
                     "traffic": (tr or {}).get("advance_sweep", {}).get("dram_bytes_per_launch") if tr else None,
                     "ncu_dram_pct_of_peak": (tr or {}).get("advance_sweep", {}).get("ncu_dram_pct_of_peak") if tr else None,
                     "bytes_per_launch": D["bytes"] / D["launches"], "ms_per_launch": D["ms"] / D["launches"],
                     "launches": D["launches"], "share_of_step": D["ms"] / ms_d if ms_d else None,
                     "push_only_gteps_host_loop": sum(ms_of[s] for s in d_roots) / (ms_d / 1e3) / 1e9,
                     "measured_in": f"push-only BFS (direction optimisation off) from {len(d_roots)} of the roots, "
                                    "host-driven loop, CUDA events per launch on the launching stream"}

    # ---- end to end through the C ABI with host buffers ----
    e2e = None
    if args.e2e_steps > 0:
        level_h = torch.empty(g.n, dtype=torch.int32, pin_memory=True)
        e_roots = [int(roots[i % len(roots)]) for i in range(args.e2e_steps)]
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for s in e_roots:
            Gh = sg.graph_load_csr(rp_h, ci_h, stream=stream)       # H2D of the step's input
            sg.run_bfs(Gh, s, level, o)
            level_h.copy_(level, non_blocking=True)                 # D2H of the step's result
            Gh.free()
        b.record(stream)
        torch.cuda.synchronize()
        e_ms = torch.tensor([a.elapsed_time(b)], dtype=torch.float64, device=dev)
        e_edges = torch.tensor([sum(ms_of[s] for s in e_roots)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(e_ms, op=dist.ReduceOp.MAX)
            dist.all_reduce(e_edges, op=dist.ReduceOp.SUM)
        e2e = {"value": float(e_edges.item()) / (float(e_ms.item()) / 1e3) / 1e9, "unit": UNIT,
               "h2d_bytes_per_step": int(rp_h.numel() * 8 + ci_h.numel() * 4),
               "d2h_bytes_per_step": int(g.n * 4), "steps": args.e2e_steps,
               "what": "per step: graph_load_csr from pinned host CSR + run_bfs + level D2H + graph_free"}
        # the paper's own methodology keeps the graph resident: per step only the root goes
        # in (ctrl block H2D from pinned memory inside run_bfs) and the level array comes out
        r_roots = [int(roots[i % len(roots)]) for i in range(args.steps)]
        for s in r_roots[:2]:
            if s not in ms_of:
                sg.run_bfs(G, s, level, o)
                ms_of[s] = m_s_of(level, deg)
        r_roots = [s for s in r_roots if s in ms_of]
        torch.cuda.synchronize()
        a.record(stream)
        for s in r_roots:
            sg.run_bfs(G, s, level, o)
            level_h.copy_(level, non_blocking=True)
        b.record(stream)
        torch.cuda.synchronize()
        e2e["graph_resident"] = {
            "value": sum(ms_of[s] for s in r_roots) / (a.elapsed_time(b) / 1e3) / 1e9 * (world if world > 1 else 1),
            "unit": UNIT, "h2d_bytes_per_step": 128, "d2h_bytes_per_step": int(g.n * 4), "steps": len(r_roots)}

    # ---- CPU baseline: the oracle, untuned, on rank 0 at N = 1 ----
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        import oracle
        t0 = time.perf_counter()
        done, edges_cpu = 0, 0
        while done == 0 or (time.perf_counter() - t0 < args.cpu_seconds and done < len(roots)):
            lv = oracle.bfs(g, int(roots[done]))
            edges_cpu += int(g.degrees()[lv != 0xFFFFFFFF].sum()) // 2
            done += 1
        dt = time.perf_counter() - t0
        cpu = {"value": edges_cpu / dt / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"{done} BFS root(s) of the same graph, single-threaded queue BFS ({dt:.1f} s)"}

    if rank == 0:
        avg = {k: statistics.mean(s[k] for s in stats) for k in ("iterations", "push_steps", "pull_steps",
                                                                 "arcs_pushed", "arcs_pulled")}
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
                "config": dict(workload_config(args, g, world), graph_gen_s=round(t_gen, 1)),
                "roofline": roofline, "roofline_dense_push": dense, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": int(launches),
                "clocks": clk.summary(), "per_step": avg}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
