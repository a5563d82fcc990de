#!/usr/bin/env python
"""A/B bench runner (replaces the round-1 one-off variant shell scripts).

Runs bench.py once per arm, R rounds interleaved (so box-level drift hits every arm alike), and
prints one summary line per run: GTEPS, ms/step, per-class ms / launches, dominant-kernel frac.

An arm is NAME=SPEC where SPEC is a ';'-separated list of
    env:VAR=VALUE        environment variable for the run (e.g. env:SG_SWEEP_FRAC64=16)
    lib:PATH             SYGRAPH_LIB override (a variant built with _build.build(defines=..., lib=...))
    define:MACRO=VALUE   build a variant library with this -D macro first (repeatable)
    arg:--flag=value     extra bench.py argument (repeatable), e.g. arg:--direction=push

    python scripts/abtest.py -R 2 base= "a14b48=arg:--beta=48" "word64=define:SG_PULL_WORD_MAX=64"
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def parse_arm(text):
    name, _, spec = text.partition("=")
    arm = {"name": name, "env": {}, "lib": None, "defines": [], "args": []}
    for item in filter(None, spec.split(";")):
        kind, _, val = item.partition(":")
        if kind == "env":
            k, _, v = val.partition("=")
            arm["env"][k] = v
        elif kind == "lib":
            arm["lib"] = val
        elif kind == "define":
            arm["defines"].append(val)
        elif kind == "arg":
            arm["args"].append(val)
        else:
            raise SystemExit(f"unknown arm item {item!r}")
    return arm


def summary(name, line):
    d = json.loads(line)
    r = d.get("roofline") or {}
    cls = {k: (round(v["ms"], 2), v["launches"]) for k, v in (r.get("classes") or {}).items() if v["launches"]}
    return (f"{name:16s} {d['value']:9.1f} {d['unit']} {d['ms_per_step']:.3f} ms/step "
            f"frac {r.get('frac', 0):.3f} {cls} clk {d.get('clocks', {}).get('sm_mhz')}")


def main():
    p = argparse.ArgumentParser()
    p.add_argument("-R", type=int, default=1, help="interleaved rounds")
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "abtest.txt"))
    p.add_argument("arms", nargs="+")
    a = p.parse_args()
    arms = [parse_arm(t) for t in a.arms]
    from paper_conf_icpp_carocc25_b200 import _build
    for arm in arms:
        if arm["defines"]:
            lib = os.path.join(ROOT, "build", "variants", arm["name"], "libsygraph.so")
            _build.build(defines=tuple(arm["defines"]), lib=lib)
            arm["lib"] = lib
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "w") as out:
        for _ in range(a.R):
            for arm in arms:
                env = dict(os.environ, **arm["env"])
                if arm["lib"]:
                    env["SYGRAPH_LIB"] = arm["lib"]
                cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--steps", str(a.steps), "--warmup",
                       str(a.warmup), "--e2e-steps", "0", "--no-cpu-baseline", "--dense-roots", "0", *arm["args"]]
                r = subprocess.run(cmd, env=env, capture_output=True, text=True)
                lines = [x for x in r.stdout.splitlines() if x.startswith("{")]
                msg = summary(arm["name"], lines[-1]) if lines else f"{arm['name']:16s} FAILED rc={r.returncode} " \
                                                                     f"{r.stderr[-300:]!r}"
                print(msg, flush=True)
                out.write(msg + "\n")


if __name__ == "__main__":
    main()
