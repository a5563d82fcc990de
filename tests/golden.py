"""Readers for tests/golden fixtures (each fixture cites its source in its header)."""
import os

import numpy as np

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def twolayer_example():
    n, active, w1, w2 = None, [], {}, {}
    with open(os.path.join(GOLDEN, "twolayer_bitmap_n8200.txt")) as f:
        for line in f:
            t = line.split()
            if not t or t[0].startswith("#"):
                continue
            if t[0] == "n":
                n = int(t[1])
            elif t[0] == "active":
                active = [int(x) for x in t[1:]]
            elif t[0] == "w1":
                w1[int(t[1])] = int(t[2], 16)
            elif t[0] == "w2":
                w2[int(t[1])] = int(t[2], 16)
    nw1 = (n + 63) // 64
    nw2 = (nw1 + 63) // 64
    words = np.zeros(nw1, np.uint64)
    for k, x in w1.items():
        words[k] = np.uint64(x)
    summ = np.zeros(nw2, np.uint64)
    for k, x in w2.items():
        summ[k] = np.uint64(x)
    return n, np.array(active, np.int64), words, summ
