"""Per-superstep device time of the device-driven (CUDA-graph) BFS on a config graph, from the
decision timestamps the last CTA of every superstep records (sg_bfs_trace; globaltimer).

    python scripts/bfs_trace.py [--config 4] [--roots 8] [--env SG_SPARSE=0 ...] [--json out.jsonl]

Prints one table per root (superstep, kind, input words / n_f / m_f, us) and the mean time per
kind over all roots; --env runs the same roots once per listed environment setting."""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icpp_carocc25_b200 as sg  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=4)
    ap.add_argument("--roots", type=int, default=8)
    ap.add_argument("--env", nargs="*", default=[""])
    ap.add_argument("--json", default=None)
    ap.add_argument("--quiet", action="store_true")
    ap.add_argument("--alpha", type=float, default=5.0)
    ap.add_argument("--beta", type=float, default=48.0)
    ap.add_argument("--segmented", type=int, default=0)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    g = gen.make_config_graph(a.config)
    roots = [int(r) for r in gen.config_sources(a.config, g)[: a.roots]]
    G = sg.graph_load_csr(g.row_ptr, g.col_idx, g.weights)
    lv = torch.empty(g.n, dtype=torch.int32, device="cuda")
    out = open(a.json, "w") if a.json else None
    for env in a.env:
        saved = dict(os.environ)
        for kv in filter(None, env.split(",")):
            k, _, v = kv.partition("=")
            os.environ[k] = v
        o = sg.opts(alpha=a.alpha, beta=a.beta, segmented=a.segmented)
        for r in roots[:2]:
            sg.run_bfs(G, r, lv, o)   # warm-up (graph instantiation)
        per_kind, totals = {}, []
        for r in roots:
            _, st = sg.run_bfs(G, r, lv, o)
            tr = sg.bfs_trace(G)
            totals.append(st.device_ms * 1e3)
            dbg = sg.ctrl_debug(G)
            if dbg[15]:
                names = ["clear", "words", "gsync1", "heavy", "flush", "gsync2", "decide", "gsync3"]
                print(f"   fused sparse loop: {dbg[15]} supersteps; us per phase: " +
                      " ".join(f"{nm} {dbg[i] / 1e3 / dbg[15]:.2f}" for i, nm in enumerate(names)))
            if not a.quiet:
                print(f"[{env or 'default'}] root {r}: {st.device_ms * 1e3:.1f} us, {len(tr)} supersteps")
                for t in tr:
                    print(f"   {t['step']:2d} {t['kind']:6s} words {t['words']:8d} nf {t['nf']:9d} mf {t['mf']:11d} "
                          f"{t['us']:8.1f} us")
            for t in tr:
                per_kind.setdefault(t["kind"], []).append(t["us"])
                if out:
                    out.write(json.dumps(dict(t, env=env, root=r)) + "\n")
        os.environ.clear()
        os.environ.update(saved)
        print(f"[{env or 'default'}] mean BFS {statistics.mean(totals):.1f} us; per kind: " +
              ", ".join(f"{k} {statistics.mean(v):.1f} us x{len(v) / len(roots):.2f}" for k, v in sorted(per_kind.items())),
              flush=True)


if __name__ == "__main__":
    main()
