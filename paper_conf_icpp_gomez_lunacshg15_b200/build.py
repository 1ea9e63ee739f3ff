"""Build libds.so (the C-ABI hot path) in-tree with nvcc for sm_100a.

    python -m paper_conf_icpp_gomez_lunacshg15_b200.build [--force] [--variant NAME]

Objects go to build/<variant>/, the library to
paper_conf_icpp_gomez_lunacshg15_b200/lib/libds[<suffix>].so (a directory of
its own so Python never mistakes it for an extension module).  Variants:
  release : -O3 -lineinfo                            -> libds.so
  stress  : -DDS_DEBUG_DELAY (random per-CTA delays) -> libds_stress.so
  strict  : -DDS_STRICT_ORDER (release/acquire status ordering) -> libds_strict.so
  spincap : -DDS_SPIN_CAP_NS (waits trap after 2 s: failure detection) -> libds_spincap.so
  hang    : spincap + -DDS_DEBUG_DROP_TILE=5 (a lost tile; test only) -> libds_hang.so
The CUDA runtime is linked statically so the library does not depend on
which libcudart the host process (torch) has loaded.
"""
from __future__ import annotations

import argparse
import concurrent.futures as cf
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
SOURCES = ["ds_api.cu", "ds_irregular.cu", "ds_regular.cu", "ds_regular_bytes.cu", "ds_shard.cu"]
HEADERS = ["ds_device.cuh", "ds_internal.h"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
VARIANTS = {
    "release": ("libds.so", []),
    "stress": ("libds_stress.so", ["-DDS_DEBUG_DELAY=1"]),
    "strict": ("libds_strict.so", ["-DDS_STRICT_ORDER=1"]),
    # failure detection: every wait traps after 2 s (no false positive expected)
    "spincap": ("libds_spincap.so", ["-DDS_SPIN_CAP_NS=2000000000ull"]),
    # the same with tile 5 of every irregular launch never publishing (test only)
    "hang": ("libds_hang.so", ["-DDS_SPIN_CAP_NS=200000000ull", "-DDS_DEBUG_DROP_TILE=5u"]),
    # irregular shared-memory layouts at the edges (tests): no output ring (every
    # tile compacted in place), a ring of about one tile (wrap-around skips and a
    # mix of ring / in place), and two input stages
    "ring0": ("libds_ring0.so", ["-DDS_IRR_RING_WORDS=0"]),
    "ring8k": ("libds_ring8k.so", ["-DDS_IRR_RING_WORDS=8704"]),
    "stages2": ("libds_stages2.so", ["-DDS_IRR_IN_STAGES=2", "-DDS_IRR_PART_STAGES=2"]),
}


def nvcc() -> str:
    for cand in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc"):
        if cand and os.path.exists(cand):
            return cand
    return "nvcc"


LIBDIR = os.path.join(PKG, "lib")


def lib_path(variant: str = "release") -> str:
    return os.path.join(LIBDIR, VARIANTS[variant][0])


def _newest_dep_mtime() -> float:
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [os.path.join(INCLUDE, "ds.h"),
                                                                   os.path.abspath(__file__)]
    return max(os.path.getmtime(d) for d in deps)


def build(variant: str = "release", force: bool = False, verbose: bool = False,
          extra_flags: list[str] | None = None, out_name: str | None = None) -> str:
    """Build one variant; extra_flags/out_name build ad-hoc tuning variants."""
    out = os.path.join(LIBDIR, out_name) if out_name else lib_path(variant)
    if not force and os.path.exists(out) and os.path.getmtime(out) >= _newest_dep_mtime():
        return out
    extra = VARIANTS[variant][1] + list(extra_flags or [])
    objdir = os.path.join(ROOT, "build", out_name.replace(".so", "") if out_name else variant)
    os.makedirs(objdir, exist_ok=True)
    os.makedirs(LIBDIR, exist_ok=True)
    common = [nvcc(), *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC",
              "-Xptxas", "-v", "-I", INCLUDE, "-I", CSRC, *extra]

    def compile_one(src: str) -> str:
        obj = os.path.join(objdir, src.replace(".cu", ".o"))
        cmd = common + ["-c", os.path.join(CSRC, src), "-o", obj]
        r = subprocess.run(cmd, capture_output=True, text=True)
        with open(obj + ".ptxas.log", "w") as fh:
            fh.write(r.stdout + r.stderr)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr}")
        if verbose:
            print(r.stderr, file=sys.stderr)
        return obj

    with cf.ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        objs = list(ex.map(compile_one, SOURCES))
    tmp = out + ".tmp"
    subprocess.check_call([nvcc(), *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs])
    os.replace(tmp, out)
    return out


def main() -> None:
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("--verbose", action="store_true")
    ap.add_argument("--variant", default="release", choices=sorted(VARIANTS))
    ap.add_argument("-D", action="append", default=[], help="extra -D for a tuning build")
    ap.add_argument("--out", default=None, help="library file name for a tuning build")
    a = ap.parse_args()
    print(build(a.variant, a.force, a.verbose, [f"-D{d}" for d in a.D], a.out))


if __name__ == "__main__":
    main()
