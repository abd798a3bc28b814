"""bench.py's reference arm (the CPU oracle on a bounded sample) and its JSON-line contract, on CPU.

The driver runs `bench.py --impl reference` beside our arm and divides the two `value`s, so the
reference line must carry the same metric, unit and config as our arm's line for that workload.
"""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def _run(*argv, env=None):
    e = dict(os.environ)
    e.update(env or {})
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", *argv],
                         capture_output=True, text=True, timeout=600, env=e, cwd=ROOT)
    assert out.returncode == 0, out.stderr
    return [json.loads(l) for l in out.stdout.splitlines() if l.startswith("{")]


def _args(workload, *extra):
    return bench.parse(["--workload", workload, *extra])


@pytest.mark.parametrize("workload,unit", [("default", "GB/s"), ("cfg3", "GB/s"), ("sweep", "trials/s"),
                                           ("trace", "warp-evaluations/s"), ("tile", "GB/s")])
def test_reference_line(workload, unit):
    (line,) = _run("--workload", workload, "--steps", "1", "--warmup", "1")
    assert line["impl"] == "reference" and line["metric"] == bench.METRIC
    assert line["unit"] == unit and line["value"] > 0 and line["higher_is_better"] is True
    assert line["config"] == bench.arm_config(_args(workload, "--steps", "1", "--warmup", "1"), 1)
    cb = line["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["value"] == line["value"] and cb["cores"] >= 1 and cb["sample"]
    assert cb["nproc"] >= 1 and "cpu_model" in cb
    assert line["e2e"] == {"value": line["value"], "unit": unit, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}
    if workload in ("default", "cfg3"):
        assert line["sweep"]["trials_per_s"] > 0
    if workload == "default":
        assert line["dtype"] == "u64" and line["config"]["rows"] == 16384 and line["config"]["elem_bytes"] == 8


def test_reference_only_rank0_prints():
    # under torchrun only rank 0 runs the oracle; the other ranks exit 0 without output
    assert _run("--steps", "1", "--warmup", "1", env={"WORLD_SIZE": "2", "RANK": "1", "LOCAL_RANK": "1"}) == []


@pytest.mark.parametrize("workload", ["default", "cfg3", "cfg4", "dist", "dist_fused", "layouts"])
def test_arm_config_bytes(workload):
    cfg = bench.arm_config(_args(workload), 4)
    n, eb = cfg["rows"], cfg["elem_bytes"]
    rows_rank = n // 4 if workload.startswith("dist") else n
    assert cfg["algorithmic_bytes_per_step_per_rank"] == 2 * rows_rank * n * eb
    assert ("4 GPU" in cfg["workload"]) == workload.startswith("dist")


def test_default_sweeps_1e9_trials():
    # the default run sweeps cfg2's 10^9 trials: a small slice per timed step (so the cfg4
    # transpose stays the step's dominant kernel) and the rest in one timed sub-run
    for k in (1, 3, 7, 20, 50):
        a = _args("default", "--steps", str(k))
        assert a.sweep_trials == bench.STEP_SWEEP_TRIALS and a.sweep_trials * k < bench.SWEEP_TOTAL
        assert bench.arm_config(a, 1)["sweep_trials_total"] == bench.SWEEP_TOTAL


def test_oracle_band_is_one_definition():
    # both arms time the oracle on the same row band of the matrix
    assert bench.oracle_band(16384, 16384, 8) == 256 and bench.oracle_band(8192, 8192, 4) == 1024
    assert bench.oracle_band(32, 32, 4) == 32


def test_golden_1e9_histogram_loads():
    h = bench.golden_sweep_1e9(1)
    assert h.shape == (5, 3, 33) and (h.sum(-1) == 10 ** 9).all()
