"""T6: performance regression guard.  Loose floors, well under the
measured numbers (compaction 256M-1G ~80-84 %, pad at 268M
elements ~100 % of the measured copy peak), so that only a real regression --
not run-to-run noise -- fails: compaction / select / unique at >= 256M words
and pad / unpad at 268M elements, min over 5 flushed launches."""
import json
import os

import pytest
import torch

import dsgen
from paper_conf_icpp_gomez_lunacshg15_b200 import libds

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _peak():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as fh:
            return float(json.load(fh)["hbm_gbs"])
    except Exception:
        return 6547.8


def _best_gbs(src, call, nbytes_fn, reps=5):
    flush = torch.empty(1 << 27, dtype=torch.int32, device="cuda")
    work = torch.empty_like(src)
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    best = None
    for r in range(reps + 2):
        work.copy_(src)
        flush.sum()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        call(work, d_n)
        b.record()
        b.synchronize()
        if r >= 2:
            t = a.elapsed_time(b) * 1e-3
            best = t if best is None else min(best, t)
    return nbytes_fn(int(d_n.item())) / best / 1e9


@pytest.mark.parametrize("op,f,floor", [("compact", 0.5, 0.70), ("compact", 0.1, 0.65), ("select", 0.0, 0.70),
                                        ("unique", 0.5, 0.65)])
def test_irregular_floor(op, f, floor):
    n = 1 << 28
    if op == "compact":
        src = dsgen.compact_input(n, f, dsgen.seed_for(3, int(f * 10)), device="cuda")
        call = lambda w, d: libds.ds_compact_ex(w, n, 0, d, None)  # noqa: E731
    elif op == "select":
        src = dsgen.select_input(n, dsgen.seed_for(2), device="cuda")
        t = dsgen.select_threshold(f) & 0xFFFFFFFF
        call = lambda w, d: libds.ds_select_ex(w, n, libds.DS_PRED_I32_GT, t, d, None)  # noqa: E731
    else:
        src = dsgen.unique_runs_input(n, f, dsgen.seed_for(2, 16), device="cuda")
        call = lambda w, d: libds.ds_unique_ex(w, n, None, 0, d, None)  # noqa: E731
    gbs = _best_gbs(src, call, lambda m: 4 * (n + m))
    assert gbs >= floor * _peak(), f"{op} f={f}: {gbs:.0f} GB/s < {floor:.0%} of {_peak():.0f}"


@pytest.mark.parametrize("op", ["pad", "unpad"])
def test_regular_floor(op):
    R, C, NC = 16384, 16383, 16384
    src = dsgen.matrix_input(R, C, NC, 4, device="cuda")
    if op == "pad":
        call = lambda w, d: libds.ds_pad_ex(w, R, C, NC, 4, None, None)  # noqa: E731
        nb = 4 * (R * C + R * NC)
    else:
        call = lambda w, d: libds.ds_unpad_ex(w, R, NC, C, 4, None)  # noqa: E731
        nb = 4 * 2 * R * C
    gbs = _best_gbs(src, call, lambda m: nb)
    assert gbs >= 0.85 * _peak(), f"{op}: {gbs:.0f} GB/s"
