"""The irregular kernel's shared-memory layout at its edges:
no output ring (every tile compacted in place), a ring of about one tile
(wrap-around skips, ring and in-place tiles mixed) and only two input stages.
The release library's parity tests for compact / select / unique / partition
/ 8-byte elements / tile edges run against each build in a subprocess."""
import os
import subprocess
import sys

import pytest

from paper_conf_icpp_gomez_lunacshg15_b200 import build

HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.mark.gpu
@pytest.mark.slow
@pytest.mark.parametrize("variant", ["ring0", "ring8k", "stages2"])
def test_irregular_parity_on_layout_variant(variant):
    lib = build.build(variant)
    env = dict(os.environ, LIBDS_PATH=lib)
    cmd = [sys.executable, "-m", "pytest", os.path.join(HERE, "test_parity_gpu.py"), "-x", "-q", "-p",
           "no:cacheprovider", "-k", "compact or select or unique or partition or 64 or edges or structured"]
    r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=1800, cwd=os.path.dirname(HERE))
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
    assert " passed" in r.stdout
