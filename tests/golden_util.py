"""Loader for tests/golden/*.txt worked examples (key: value lines, # comments)."""
import glob
import os

import numpy as np

GOLDEN_DIR = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
_LIST_KEYS = {"input", "output", "buffer_after"}


def load(path):
    d = {}
    with open(path) as fh:
        for line in fh:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, v = line.split(":", 1)
            k, v = k.strip(), v.strip()
            if k in _LIST_KEYS:
                d[k] = np.array([int(x) & 0xFFFFFFFF for x in v.split()], dtype=np.uint32)
            elif k == "op":
                d[k] = v
            else:
                d[k] = int(v)
    d["name"] = os.path.basename(path)
    return d


def all_cases():
    return [load(p) for p in sorted(glob.glob(os.path.join(GOLDEN_DIR, "*.txt")))]
