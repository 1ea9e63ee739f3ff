"""bench.py contract: the reference arm on CPU (any box) and, on a GPU, the
libds arm's JSON line with its required keys -- plain and under torchrun with
one process, which must print the same schema."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BASE_KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
             "scaling", "vs_baseline", "dtype", "data", "config", "e2e"}


def _json_line(out):
    lines = [ln for ln in out.splitlines() if ln.startswith("{")]
    assert lines, out[-2000:]
    return json.loads(lines[-1])


def test_reference_arm_on_cpu():
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                        "--warmup", "0"], capture_output=True, text=True, timeout=600, env=env, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    d = _json_line(r.stdout)
    assert BASE_KEYS <= set(d), set(d)
    assert d["impl"] == "reference" and d["unit"] == "GB/s" and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] == 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0
    sys.path.insert(0, ROOT)
    import bench
    assert d["config"] == bench.bench_config(1, "collective")   # the same config dict as the libds arm


def _libds_line(cmd):
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=1200, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    return _json_line(r.stdout)


@pytest.mark.gpu
@pytest.mark.slow
def test_libds_arm_schema_plain_and_torchrun():
    args = ["--steps", "3", "--warmup", "3", "--no-rows", "--no-cpu", "--e2e-steps", "1"]
    plain = _libds_line([sys.executable, os.path.join(ROOT, "bench.py"), *args])
    tr = _libds_line([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "1",
                      "--master-addr", "127.0.0.1", "--master-port", "29517", os.path.join(ROOT, "bench.py"),
                      "--gpus", "1", *args])
    for d in (plain, tr):
        assert BASE_KEYS <= set(d)
        assert {"roofline", "clocks", "gpu_launches", "per_rank", "kernel_ms_max", "collective_ms_max",
                "step_stats_rank0"} <= set(d)
        rf = d["roofline"]
        assert rf["bound"] == "hbm" and rf["unit"] == "GB/s" and 0 < rf["frac"] < 1.2
        assert d["gpu_launches"] == 2 * d["steps"]      # ds_compact_ex + ds_shard_offsets per step
        assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert set(plain) == set(tr)                        # same schema under torchrun
    assert set(plain["roofline"]) == set(tr["roofline"])
    assert plain["config"] == tr["config"]
    sys.path.insert(0, ROOT)
    import bench
    assert plain["config"] == bench.bench_config(1, "collective")   # what the reference arm reports


@pytest.mark.gpu
@pytest.mark.slow
@pytest.mark.parametrize("exchange", ["collective", "board"])
def test_libds_arm_two_ranks_logic(exchange):
    """The N > 1 logic of bench.py (per-rank kernel / collective times, max over
    ranks, whole-job value, e2e, the rebalance leg) with 2 ranks on this one GPU:
    test mode (DS_BENCH_TEST_GLOO) runs them over gloo with host-staged
    collectives and a 2^24-word array -- NCCL itself needs one GPU per rank."""
    env = dict(os.environ, DS_BENCH_TEST_GLOO="1", DS_BENCH_N_LOG2="24")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", "29519", os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--steps", "3", "--warmup", "3", "--no-rows", "--no-cpu", "--e2e-steps", "1",
           "--rebalance", "--count-exchange", exchange]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-4000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]                    # rank 0 alone prints
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and len(d["per_rank"]) == 2 and d["config"]["n_total"] == 1 << 24
    assert d["config"]["count_exchange"] == exchange and "TEST MODE" in d["config"]["workload"]
    assert d["value"] > 0 and d["kernel_ms_max"] > 0 and d["collective_ms_max"] >= 0
    assert d["rebalance"]["ms"] > 0 and d["e2e"]["value"] > 0
