"""T3: scheduling stress with the delay-injection build (libds_stress.so)."""
import os
import subprocess
import sys

import pytest

from paper_conf_icpp_gomez_lunacshg15_b200 import build

HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.mark.gpu
@pytest.mark.parametrize("variant", ["stress", "strict"])
def test_delay_injection_parity(variant):
    """stress: random per-CTA delays (-DDS_DEBUG_DELAY); strict: the
    release/acquire status ordering build (-DDS_STRICT_ORDER)."""
    lib = build.build(variant)
    env = dict(os.environ, LIBDS_PATH=lib)
    r = subprocess.run([sys.executable, os.path.join(HERE, "stress_driver.py"), "12"],
                       env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]
    assert "stress OK" in r.stdout


@pytest.mark.gpu
@pytest.mark.slow
@pytest.mark.parametrize("variant", ["stress", "strict", "release"])
def test_relaxed_ordering_full_size(variant):
    """The relaxed status ordering (R10) at full size: 50 launches each of
    256M-word compaction at f = 0.1 / 0.5 / 0.9 and unique, with random
    per-CTA delays (stress) and in the release build, all bit-exact."""
    lib = build.build(variant)
    env = dict(os.environ, LIBDS_PATH=lib)
    r = subprocess.run([sys.executable, os.path.join(HERE, "stress_driver.py"), "50", "large"],
                       env=env, capture_output=True, text=True, timeout=1800)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]
    assert "stress OK: large" in r.stdout
