#!/usr/bin/env python
"""bench.py — BFS GTEPS on the config-4 workload (Kronecker/R-MAT scale 24, edge factor 32,
permuted, direction-optimising), through the C ABI of libsygraph.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl sygraph|reference] [--config 4]

One *step* = one full BFS (all §8(a) rows: compaction, tiered push / pull advance, frontier
swap/clear, direction policy) from one of the 64 seeded roots.  `value` = Graph500 TEPS of the
K timed roots / max-over-ranks device time (CUDA events, barrier + synchronize on both sides).
N > 1 (torchrun, one process per GPU): the graph is 1-D destination-partitioned over the ranks
(graph_load_csr with a communicator) and every BFS is one collective run whose
supersteps exchange the owned frontier slices over NVLink peer memory inside the output kernels
(strong scaling: the same graph and roots at every N; each rank keeps its owned part of the
level array, Graph500-style — the result gather is outside the timed region, in `e2e`).
The graph (4 GB of col_idx) is larger than L2, so no flush is needed.  Extra lines in the same
JSON object: per-root median / Graph500 harmonic mean, config-2 SSSP GTEPS (`sssp_c2`) and
config-3 CC (`cc_c3`), both on the same N GPUs.  `e2e` = the same metric through
graph_load_csr from pinned HOST buffers + run_bfs + level D2H per step.  `--impl reference`
times the oracle (queue BFS, one host core) on the same workload.
SG_BENCH_SHARE_GPU=1 runs every rank on cuda:0 (gloo process group): a functional check of the
N > 1 path on a one-GPU box (time-sliced, so its numbers are not a measurement).
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
    p.add_argument("--alpha", type=float, default=5.0)
    p.add_argument("--beta", type=float, default=48.0)
    p.add_argument("--heavy-degree", type=int, default=0, help="CTA/grid-tier degree threshold (0: library default)")
    p.add_argument("--scsr", type=int, default=0, help="segmented push advance: 0 auto, 1 off, 2 always")
    p.add_argument("--e2e-steps", type=int, default=3)
    p.add_argument("--dense-roots", type=int, default=3, help="push-only BFS roots for roofline_dense_push (0: skip)")
    p.add_argument("--cpu-seconds", type=float, default=15.0)
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--extra-steps", type=int, default=10, help="repetitions of the C2 SSSP / C3 CC lines (0: skip)")
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


def shared_graph(cfg, seed, R, rank, pinned=False):
    """N > 1: rank 0 generates the config graph and hands it to the other ranks through /dev/shm
    (one generator run instead of N concurrent ones competing for the host cores); every rank
    gets its own copy (pinned if asked).  N = 1: plain generation."""
    import gen
    if R.world == 1:
        return make_graph(cfg, seed, pinned) if pinned else gen.make_config_graph(cfg, seed=seed)
    import torch
    tag = f"/dev/shm/sygraph_bench_{os.environ.get('MASTER_PORT', '0')}_{cfg}_{seed}"
    if rank == 0:
        g = make_graph(cfg, seed, pinned) if pinned else gen.make_config_graph(cfg, seed=seed)
        g.row_ptr.tofile(tag + ".rp")
        g.col_idx.tofile(tag + ".ci")
        if g.weights is not None:
            g.weights.tofile(tag + ".w")
        with open(tag + ".meta", "w") as f:
            json.dump({"n": g.n, "name": g.name}, f)
    R.barrier()
    if rank != 0:
        meta = json.load(open(tag + ".meta"))
        rp = np.fromfile(tag + ".rp", dtype=np.int64)
        ci = np.fromfile(tag + ".ci", dtype=np.int32)
        w = np.fromfile(tag + ".w", dtype=np.uint8) if os.path.exists(tag + ".w") else None
        keep = {}
        if pinned:
            rp_t = torch.empty(len(rp), dtype=torch.int64, pin_memory=True)
            ci_t = torch.empty(max(len(ci), 1), dtype=torch.int32, pin_memory=True)
            rp_t.numpy()[:] = rp
            ci_t.numpy()[:len(ci)] = ci
            keep = {"rp": rp_t, "ci": ci_t}
            rp, ci = rp_t.numpy(), ci_t.numpy()[:len(ci)]
        g = gen.CSR(n=meta["n"], row_ptr=rp, col_idx=ci, name=meta["name"], weights=w)
        g.meta["pinned"] = keep
    R.barrier()
    if rank == 0:
        for ext in (".rp", ".ci", ".w", ".meta"):
            if os.path.exists(tag + ext):
                os.unlink(tag + ext)
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
            "parallelism": (f"1-D destination partition over {world} GPUs (peer-memory exchange)"
                            if world > 1 else "1 GPU"),
            "l2": "inputs larger than L2 (4 GB col_idx vs 126 MB L2)"}


def host_cpu():
    """nproc and the CPU model of this host (for the oracle baseline)."""
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name:"):
                model = line.split(":", 1)[1].strip()
    except Exception:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model}


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
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": workload_config(args, g, args.gpus),
            "cpu_baseline": dict({"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                                  "sample": f"{args.steps} timed queue-BFS roots (1 BFS per step)"}, **host_cpu()),
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


class Ranks:
    """torch.distributed plumbing: barrier and max / sum over ranks (nccl on one GPU per rank,
    gloo when SG_BENCH_SHARE_GPU puts every rank on cuda:0)."""

    def __init__(self, world, local):
        import torch
        import torch.distributed as dist
        self.world, self.dist, self.torch = world, dist, torch
        self.rank = int(os.environ.get("RANK", "0"))
        self.share = os.environ.get("SG_BENCH_SHARE_GPU") == "1"
        self.dev = torch.device("cuda", 0 if self.share else local)
        torch.cuda.set_device(self.dev)
        if world > 1:
            if self.share:
                dist.init_process_group("gloo")
            else:
                dist.init_process_group("nccl", device_id=self.dev)
        self.tdev = torch.device("cpu") if self.share else self.dev

    def barrier(self):
        if self.world > 1:
            self.dist.barrier()

    def reduce(self, x, op):
        if self.world == 1:
            return float(x)
        t = self.torch.tensor([float(x)], dtype=self.torch.float64, device=self.tdev)
        self.dist.all_reduce(t, op=self.dist.ReduceOp.MAX if op == "max" else self.dist.ReduceOp.SUM)
        return float(t.item())

    def close(self):
        if self.world > 1:
            self.dist.destroy_process_group()


def extra_lines(args, R, comm, sg, torch, stream):
    """C2 SSSP GTEPS and C3 CC time on the same N GPUs (device-resident, max over ranks)."""
    out = {}
    if args.extra_steps <= 0:
        return out
    # ---- C2: SSSP, integer weights 1..64, RMAT-20 EF16, from vertex 0 ----
    g2 = shared_graph(2, args.seed, R, R.rank)
    G2 = sg.graph_load_csr(g2.row_ptr, g2.col_idx, g2.weights, comm=comm)
    deg2 = torch.diff(torch.from_numpy(g2.row_ptr).to(R.dev))
    dist_t = torch.empty(g2.n, dtype=torch.int32, device=R.dev)
    o2 = sg.opts(stream=stream)
    sg.run_sssp(G2, 0, dist_t, o2)
    m_s = m_s_of(dist_t, deg2)
    R.barrier()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(stream)
    for _ in range(args.extra_steps):
        _, st2 = sg.run_sssp(G2, 0, dist_t, o2)
    b.record(stream)
    torch.cuda.synchronize()
    ms2 = R.reduce(a.elapsed_time(b), "max") / args.extra_steps
    out["sssp_c2"] = {"metric": "SSSP GTEPS (Graph500 m_s / time), RMAT-20 EF16, weights 1..64, source 0",
                      "value": m_s / (ms2 / 1e3) / 1e9, "unit": "GTEPS", "ms_per_run": ms2, "runs": args.extra_steps,
                      "supersteps": st2.iterations, "arcs_relaxed": st2.arcs_pushed, "n": g2.n, "nnz": g2.nnz}
    G2.free()
    del g2
    # ---- C3: CC by label propagation, uniform G(n=21M, m=265M) = 530M arcs ----
    g3 = shared_graph(3, args.seed, R, R.rank)
    G3 = sg.graph_load_csr(g3.row_ptr, g3.col_idx, comm=comm)
    lab = torch.empty(g3.n, dtype=torch.int32, device=R.dev)
    o3 = sg.opts(stream=stream)
    sg.run_cc(G3, lab, o3)
    reps = max(1, args.extra_steps // 2)
    R.barrier()
    torch.cuda.synchronize()
    a.record(stream)
    for _ in range(reps):
        _, st3 = sg.run_cc(G3, lab, o3)
    b.record(stream)
    torch.cuda.synchronize()
    ms3 = R.reduce(a.elapsed_time(b), "max") / reps
    out["cc_c3"] = {"metric": "CC label propagation, G(21M, 265M) = 530M arcs: time per run and arcs/s (nnz / time)",
                    "ms_per_run": ms3, "value": g3.nnz / (ms3 / 1e3) / 1e9, "unit": "G arcs/s", "runs": reps,
                    "supersteps": st3.iterations, "push_steps": st3.push_steps, "pull_steps": st3.pull_steps,
                    "arcs_processed": st3.arcs_pushed + st3.arcs_pulled, "n": g3.n, "nnz": g3.nnz}
    G3.free()
    return out


def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        # torchrun sets OMP_NUM_THREADS=1; rank 0 alone runs the (OpenMP) generator for all ranks
        # (shared_graph), so give it the host's cores
        os.environ["OMP_NUM_THREADS"] = str(os.cpu_count() or 8)
    if args.impl == "reference":
        return run_reference(args, rank)

    import torch
    import gen
    import paper_conf_icpp_carocc25_b200 as sg

    R = Ranks(world, local)
    dev = R.dev
    stream = torch.cuda.current_stream()
    comm = sg.comm_from_torch(device=dev.index) if world > 1 else None
    if comm is not None and rank == 0:
        print(f"[bench] partition communicator: {world} ranks, peer-memory exchange "
              f"({'shared GPU, time-sliced' if R.share else 'one GPU per rank'})", file=sys.stderr, flush=True)

    t_gen = time.perf_counter()
    g = shared_graph(args.config, args.seed, R, rank, pinned=True)
    t_gen = time.perf_counter() - t_gen
    roots = gen.config_sources(args.config, g, seed=args.seed)
    rp_h = torch.from_numpy(g.row_ptr)
    ci_h = torch.from_numpy(g.col_idx)
    t_load = time.perf_counter()
    G = sg.graph_load_csr(rp_h, ci_h, comm=comm)          # host -> device copy (not timed)
    t_load = time.perf_counter() - t_load
    lo, hi = sg.graph_partition(G)
    deg = torch.diff(rp_h.to(dev))
    direction = {"auto": sg.SG_DIR_AUTO, "push": sg.SG_DIR_PUSH, "pull": sg.SG_DIR_PULL}[args.direction]
    mk = dict(stream=stream, direction=direction, alpha=args.alpha, beta=args.beta, heavy_degree=args.heavy_degree,
              scsr=args.scsr)
    o = sg.opts(**mk, owned_only=world > 1)      # timed runs: each rank keeps its owned levels
    o_full = sg.opts(**mk)                        # result gathered on every rank (m_s, e2e)
    level = torch.empty(g.n, dtype=torch.int32, device=dev)

    # m_s per root (untimed; BFS results are deterministic per root)
    step_roots = [int(roots[(args.warmup + i) % len(roots)]) for i in range(args.steps)]
    ms_of = {}
    for s in sorted(set(step_roots) | {int(roots[i % len(roots)]) for i in range(max(args.e2e_steps, 1))}):
        sg.run_bfs(G, s, level, o_full)
        ms_of[s] = m_s_of(level, deg)
    for i in range(args.warmup):
        sg.run_bfs(G, int(roots[i % len(roots)]), level, o)

    # ---- timed region (device-resident inputs; each BFS is one CUDA graph launch) ----
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    stats = []
    R.barrier()
    torch.cuda.synchronize()
    launches0 = sg.launch_count()
    with ClockSampler(dev.index) as clk:
        ev0.record(stream)
        for s in step_roots:
            _, st = sg.run_bfs(G, s, level, o)
            stats.append(st.as_dict())
        ev1.record(stream)
        torch.cuda.synchronize()
    R.barrier()
    launches = sg.launch_count() - launches0
    ms = ev0.elapsed_time(ev1)
    ms_max = R.reduce(ms, "max")
    edges = sum(ms_of[s] for s in step_roots)
    value = edges / (ms_max / 1e3) / 1e9
    # per-root TEPS from each run's own device time (max over ranks per root)
    per_ms = [R.reduce(st["device_ms"], "max") for st in stats]
    teps = [ms_of[s] / (t / 1e3) / 1e9 for s, t in zip(step_roots, per_ms)]
    per_root = {"gteps_median": statistics.median(teps), "gteps_hmean": len(teps) / sum(1.0 / t for t in teps),
                "gteps_min": min(teps), "gteps_max": max(teps),
                "slowest_root": step_roots[int(np.argmin(teps))], "ms_max": max(per_ms), "ms_median": statistics.median(per_ms),
                "what": "Graph500 per-root TEPS (m_s / the run's device time): median and harmonic mean"}

    peak, peak_src = peaks()
    tr = committed_traffic()
    roofline = dense = None
    if world == 1:
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
        dom = max(prof, key=lambda k: prof[k]["ms"])
        P = prof[dom]
        achieved = (P["bytes"] / P["launches"]) / (P["ms"] / P["launches"] / 1e3) / 1e9 if P["launches"] else 0.0
        trd = (tr or {}).get(dom, {})
        roofline = {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": peak, "unit": "GB/s",
                    "frac": achieved / peak, "peak_source": peak_src,
                    "traffic": trd.get("dram_bytes_per_launch"),
                    "sector_efficiency": trd.get("lsu_sector_efficiency"),
                    "ncu_dram_pct_of_peak": trd.get("ncu_dram_pct_of_peak"),
                    "bytes_per_launch": P["bytes"] / max(P["launches"], 1),
                    "ms_per_launch": P["ms"] / max(P["launches"], 1),
                    "share_of_step": P["ms"] / ms_prof if ms_prof else None,
                    "measured_in": "CUDA events per launch on the launching stream, host-driven pass over the "
                                   "timed region's K roots (ms_per_step %.3f there)" % (ms_prof / args.steps),
                    "classes": {k: {"ms": v["ms"], "launches": v["launches"],
                                    "GBps": (v["bytes"] / (v["ms"] / 1e3) / 1e9) if v["ms"] else 0.0,
                                    "sector_efficiency": (tr or {}).get(k, {}).get("lsu_sector_efficiency")}
                                for k, v in prof.items()}}

        # ---- the north star's HBM bar: the dense top-down advance (direction optimisation off) ----
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
                    sg.run_bfs(G, s, level, o_full)
                    ms_of[s] = m_s_of(level, deg)
            D = dprof.get("advance_sweep", {"launches": 0})
            if D["launches"]:
                ach = (D["bytes"] / D["launches"]) / (D["ms"] / D["launches"] / 1e3) / 1e9
                trs = (tr or {}).get("advance_sweep", {})
                dense = {"bound": "hbm", "kernel": "k_push_sweep (advance_sweep)", "achieved": ach, "peak": peak,
                         "unit": "GB/s", "frac": ach / peak, "peak_source": peak_src,
                         "traffic": trs.get("dram_bytes_per_launch"),
                         "ncu_dram_pct_of_peak": trs.get("ncu_dram_pct_of_peak"),
                         "sector_efficiency": trs.get("lsu_sector_efficiency"),
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
        # one untimed warm-up step: the first load of a second graph maps fresh device memory
        Gw = sg.graph_load_csr(rp_h, ci_h, stream=stream, comm=comm)
        sg.run_bfs(Gw, e_roots[0], level, o_full)
        Gw.free()
        R.barrier()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for s in e_roots:
            Gh = sg.graph_load_csr(rp_h, ci_h, stream=stream, comm=comm)   # H2D of the step's input
            sg.run_bfs(Gh, s, level, o_full)
            level_h.copy_(level, non_blocking=True)                         # D2H of the step's result
            Gh.free()
        b.record(stream)
        torch.cuda.synchronize()
        e_ms = R.reduce(a.elapsed_time(b), "max")
        e2e = {"value": sum(ms_of[s] for s in e_roots) / (e_ms / 1e3) / 1e9, "unit": UNIT,
               "h2d_bytes_per_step": int(rp_h.numel() * 8 + ci_h.numel() * 4),
               "d2h_bytes_per_step": int(g.n * 4), "steps": args.e2e_steps,
               "what": "per step: graph_load_csr from pinned host CSR (partitioned when N > 1) + run_bfs with the "
                       "result gathered on every rank + level D2H + graph_free"}
        # the paper's own methodology keeps the graph resident: per step only the root goes
        # in (ctrl block H2D from pinned memory inside run_bfs) and the level array comes out
        r_roots = [s for s in step_roots if s in ms_of]
        R.barrier()
        torch.cuda.synchronize()
        a.record(stream)
        for s in r_roots:
            sg.run_bfs(G, s, level, o_full)
            level_h.copy_(level, non_blocking=True)
        b.record(stream)
        torch.cuda.synchronize()
        r_ms = R.reduce(a.elapsed_time(b), "max")
        e2e["graph_resident"] = {"value": sum(ms_of[s] for s in r_roots) / (r_ms / 1e3) / 1e9, "unit": UNIT,
                                 "h2d_bytes_per_step": 128, "d2h_bytes_per_step": int(g.n * 4), "steps": len(r_roots)}

    extras = extra_lines(args, R, comm, sg, torch, stream)

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
        cpu = dict({"value": edges_cpu / dt / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
                    "sample": f"{done} BFS root(s) of the same graph, single-threaded queue BFS ({dt:.1f} s)"},
                   **host_cpu())

    if rank == 0:
        avg = {k: statistics.mean(s[k] for s in stats) for k in ("iterations", "push_steps", "pull_steps",
                                                                 "arcs_pushed", "arcs_pulled")}
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
                "scaling": "strong" if world > 1 else "weak", "vs_baseline": None, "dtype": "int32",
                "data": "synthetic", "config": workload_config(args, g, world),
                "per_root": per_root, "roofline": roofline, "roofline_dense_push": dense, "cpu_baseline": cpu,
                "e2e": e2e, "gpu_launches": int(launches), "clocks": clk.summary(), "per_step": avg,
                "setup_s": {"graph_gen": round(t_gen, 1), "graph_load": round(t_load, 2)},
                "partition": {"ranks": world, "rank0_owned": [lo, hi]} if world > 1 else None, **extras}
        print(json.dumps(line), flush=True)
    if comm is not None:
        G.free()
        comm.free()
    R.close()
    return 0


if __name__ == "__main__":
    sys.exit(main())
