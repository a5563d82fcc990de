"""Build libsygraph.so tuning variants under build/variants/<name>/ (for scripts/variant_bench.sh).

    python scripts/build_variants.py name:DEF=1,DEF2=3 [name2:...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_carocc25_b200 import _build  # noqa: E402

for spec in sys.argv[1:]:
    name, defs = spec.split(":", 1)
    d = tuple(x for x in defs.split(",") if x)
    out = os.path.join(_build.ROOT, "build", "variants", name, "libsygraph.so")
    os.makedirs(os.path.dirname(out), exist_ok=True)
    _build.build(defines=d, lib=out)
    print("built", out, d)
