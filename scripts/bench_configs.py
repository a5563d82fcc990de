"""Measure every BASELINE.json configuration on one GPU (device-resident inputs, CUDA events),
next to the oracle on one host core.  Writes one JSON object per config to stdout.

    python scripts/bench_configs.py [--configs 1,2,3,4,5] [--reps 5]

C1/C4 BFS (GTEPS, Graph500 m_s), C2 SSSP (GTEPS = m_s / time, relaxed arcs reported), C3 CC
(arcs/s = nnz / time), C5 BC (time per source; sources = first 4 of the 64 by default)."""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

INF = 0xFFFFFFFF


def timed(fn, reps):
    s = torch.cuda.current_stream()
    fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(reps):
        out = fn()
    b.record(s)
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps, out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="1,2,3,4,5")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--bc-sources", type=int, default=4)
    args = ap.parse_args()
    torch.cuda.set_device(0)
    for cfg in [int(c) for c in args.configs.split(",")]:
        t0 = time.time()
        g = gen.make_config_graph(cfg)
        tgen = time.time() - t0
        G = sg.graph_load_csr(g.row_ptr, g.col_idx, g.weights)
        deg = g.degrees()
        rec = {"config": cfg, "workload": gen.CONFIGS[cfg]["workload"], "n": g.n, "nnz": g.nnz, "gen_s": round(tgen, 1)}
        if cfg in (1, 4):
            roots = gen.config_sources(cfg, g)[:8]
            ms_list, teps = [], []
            lvb = torch.empty(g.n, dtype=torch.int32, device="cuda")
            sg.run_bfs(G, int(roots[0]), lvb)   # graph build outside the timing
            for s in roots:
                # the library's own device time per run (CUDA events around its graph launch), median
                # of `reps` runs: host gaps between the calls are not BFS time (bench.py's
                # per_root uses the same)
                dts = [sg.run_bfs(G, int(s), lvb)[1].device_ms for _ in range(args.reps)]
                ms = float(np.median(dts))
                m_s = int(deg[sg.as_u32(lvb) != INF].sum()) // 2
                ms_list.append(ms)
                teps.append(m_s / (ms / 1e3) / 1e9)
            t1 = time.perf_counter()
            lv = oracle.bfs(g, int(roots[0]))
            tcpu = time.perf_counter() - t1
            m0 = int(deg[lv != INF].sum()) // 2
            rec.update(metric="BFS GTEPS", gpu_ms_median=float(np.median(ms_list)),
                       gteps_median=float(np.median(teps)), gteps_hmean=float(len(teps) / np.sum(1 / np.array(teps))),
                       oracle_s=tcpu, oracle_gteps=m0 / tcpu / 1e9, roots=len(roots))
        elif cfg == 2:
            s = 0
            _, (d, st) = timed(lambda: sg.run_sssp(G, s), 1)
            ms = float(np.median([sg.run_sssp(G, s, d)[1].device_ms for _ in range(args.reps)]))   # device time
            dd = sg.as_u32(d)
            m_s = int(deg[dd != INF].sum()) // 2
            t1 = time.perf_counter()
            oracle.sssp(g, s)
            tcpu = time.perf_counter() - t1
            rec.update(metric="SSSP GTEPS", gpu_ms=ms, gteps=m_s / (ms / 1e3) / 1e9, supersteps=st.iterations,
                       arcs_relaxed=st.arcs_pushed, oracle_s=tcpu, oracle_gteps=m_s / tcpu / 1e9)
        elif cfg == 3:
            _, (lab, st) = timed(lambda: sg.run_cc(G), 1)
            ms = float(np.median([sg.run_cc(G, lab)[1].device_ms for _ in range(max(1, args.reps // 2))]))
            t1 = time.perf_counter()
            oracle.cc(g)
            tcpu = time.perf_counter() - t1
            rec.update(metric="CC time", gpu_ms=ms, garcs_per_s=g.nnz / (ms / 1e3) / 1e9, supersteps=st.iterations,
                       arcs_processed=st.arcs_pushed, oracle_s=tcpu)
        elif cfg == 5:
            srcs = gen.config_sources(5, g)[: args.bc_sources]
            ms, (bc, st) = timed(lambda: sg.run_bc(G, srcs), 1)
            t1 = time.perf_counter()
            oracle.bc(g, srcs[:1])
            tcpu = time.perf_counter() - t1
            rec.update(metric="BC time per source", gpu_ms_per_source=ms / len(srcs), supersteps=st.iterations,
                       sources=len(srcs), oracle_s_per_source=tcpu)
        print(json.dumps(rec), flush=True)
        del G


if __name__ == "__main__":
    main()
