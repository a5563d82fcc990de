"""Offline "device inspector" (§3.2: SYgraph inspects the device to pick its
kernel parameters): query the GPU, then tune the BFS knobs on the bench workload by
coordinate descent from the library defaults (one knob at a time, median device time over the
roots of each value), and the CC label block on config 3.  Writes one JSON object.

    python scripts/autotune.py [--roots 8] [--out profiles/r02_autotune.json]

Knobs: heavy_degree (CTA/grid tier threshold), small_degree (thread tier), coarsening (words
per warp grab), alpha / beta (Beamer), SG_PULL_WARP_FRAC (late warp-owned pulls), SG_SPARSE (fused
small supersteps); CC: SG_CC_LBLOCK_KB.  No knob changes results (tested); only time."""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402

OPT_KNOBS = {"heavy_degree": [1024, 2048, 4096], "small_degree": [16, 32, 64], "coarsening": [0, 2, 4],
             "alpha": [3.0, 5.0, 8.0, 14.0], "beta": [24.0, 48.0, 96.0]}
ENV_KNOBS = {"SG_PULL_WARP_FRAC": ["0", "8", "16"], "SG_SPARSE": ["0", "1"]}
DEFAULTS = {"heavy_degree": 2048, "small_degree": 32, "coarsening": 0, "alpha": 5.0, "beta": 48.0,
            "SG_PULL_WARP_FRAC": "8", "SG_SPARSE": "0"}


def device_info():
    p = torch.cuda.get_device_properties(0)
    return {"name": p.name, "sms": p.multi_processor_count, "l2_bytes": getattr(p, "L2_cache_size", None),
            "total_mem": p.total_memory, "cc": f"{p.major}.{p.minor}"}


def time_bfs(G, roots, lv, cfg, reps):
    env = {k: cfg[k] for k in ENV_KNOBS}
    saved = {k: os.environ.get(k) for k in env}
    os.environ.update(env)
    try:
        o = sg.opts(**{k: cfg[k] for k in OPT_KNOBS})
        sg.run_bfs(G, roots[0], lv, o)   # graph (re)build
        ts = []
        for r in roots:
            best = min(sg.run_bfs(G, r, lv, o)[1].device_ms for _ in range(reps))
            ts.append(best)
        return statistics.median(ts), statistics.mean(ts)
    finally:
        for k, v in saved.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--roots", type=int, default=8)
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    out = {"device": device_info(), "workload": "config 4 BFS (Kronecker-24 EF32), device_ms per root (graph mode)"}
    g = gen.make_config_graph(4)
    roots = [int(r) for r in gen.config_sources(4, g)[: a.roots]]
    G = sg.graph_load_csr(g.row_ptr, g.col_idx)
    lv = torch.empty(g.n, dtype=torch.int32, device="cuda")
    cur = dict(DEFAULTS)
    base_med, base_mean = time_bfs(G, roots, lv, cur, a.reps)
    out["default"] = {"cfg": dict(cur), "median_ms": base_med, "mean_ms": base_mean}
    sweeps = []
    for knob, values in list(OPT_KNOBS.items()) + list(ENV_KNOBS.items()):
        res = []
        for v in values:
            cfg = dict(cur, **{knob: v})
            med, mean = time_bfs(G, roots, lv, cfg, a.reps)
            res.append({"value": v, "median_ms": med, "mean_ms": mean})
        best = min(res, key=lambda x: x["mean_ms"])
        # keep the default unless a value wins by more than 1 % (noise floor of one box)
        dflt = next(x for x in res if x["value"] == cur[knob])
        if best["mean_ms"] < 0.99 * dflt["mean_ms"]:
            cur[knob] = best["value"]
        sweeps.append({"knob": knob, "results": res, "kept": cur[knob]})
        print(json.dumps(sweeps[-1]), flush=True)
    tuned_med, tuned_mean = time_bfs(G, roots, lv, cur, a.reps)
    out["bfs_sweeps"] = sweeps
    out["tuned"] = {"cfg": cur, "median_ms": tuned_med, "mean_ms": tuned_mean,
                    "vs_default_mean": base_mean / tuned_mean}
    del G
    # CC label block (config 3)
    g3 = gen.make_config_graph(3)
    G3 = sg.graph_load_csr(g3.row_ptr, g3.col_idx)
    cc = []
    for kb in ("16384", "32768", "49152"):
        os.environ["SG_CC_LBLOCK_KB"] = kb
        sg.run_cc(G3)
        ts = [sg.run_cc(G3)[1].device_ms for _ in range(3)]
        cc.append({"SG_CC_LBLOCK_KB": kb, "median_ms": statistics.median(ts)})
    os.environ.pop("SG_CC_LBLOCK_KB", None)
    out["cc_label_block"] = cc
    text = json.dumps(out, indent=1)
    print(text)
    if a.out:
        with open(a.out, "w") as f:
            f.write(text)


if __name__ == "__main__":
    main()
