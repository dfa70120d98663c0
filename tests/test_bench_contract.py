"""bench.py's JSON-line contract (the driver parses it): the reference arm on the host
cores (CPU), the non-zero ranks of a torchrun launch of that arm, and (GPU) the default
arm's line with its roofline / e2e / clocks / launch-count fields."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BASELINE = json.load(open(os.path.join(ROOT, "BASELINE.json")))


def _run(args, env_extra=None, timeout=900):
    env = dict(os.environ, **(env_extra or {}))
    p = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], cwd=ROOT, env=env,
                       capture_output=True, text=True, timeout=timeout)
    assert p.returncode == 0, p.stderr[-3000:]
    lines = [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
    return [json.loads(ln) for ln in lines]


def _common(d, steps, warmup):
    assert d["metric"] == BASELINE["metric"]
    assert d["unit"] == "evals/s" and d["higher_is_better"] is True
    assert d["value"] > 0 and d["ms_per_step"] > 0
    assert d["n_gpus"] == 1 and d["steps"] == steps and d["warmup"] == warmup
    assert d["data"] == "synthetic" and d["vs_baseline"] is None
    assert d["scaling"] in ("weak", "strong")
    assert "workload" in d["config"] and "model" not in d["config"]
    assert d["e2e"]["value"] > 0 and d["e2e"]["unit"] == d["unit"]


def test_reference_arm_line():
    """--impl reference: the FP64 oracle on the host cores, one JSON line with the
    reference-arm fields (rank 0 of a single-process run)."""
    out = _run(["--impl", "reference", "--steps", "1", "--warmup", "3"])
    assert len(out) == 1
    d = out[0]
    _common(d, 1, 3)
    assert d["impl"] == "reference" and d["dtype"] == "f64"
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] == d["value"] and cb["sample"]
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0


def test_reference_arm_other_ranks_exit_quietly():
    """Under torchrun the reference arm runs on rank 0 only: another rank prints nothing
    and exits 0 (no process group is needed for that)."""
    out = _run(["--impl", "reference", "--gpus", "2", "--steps", "1", "--warmup", "3"],
               {"RANK": "1", "LOCAL_RANK": "1", "WORLD_SIZE": "2"})
    assert out == []


@pytest.mark.gpu
def test_default_arm_line():
    """The default arm (config 2, SIMT engine) on cuda:0: the line the driver records, with
    roofline (dominant kernel, measured live), e2e through host buffers, sampled clocks and
    the count of this library's launches."""
    out = _run(["--steps", "2", "--warmup", "3", "--no-paper-engine", "--no-lga"])
    assert len(out) == 1
    d = out[0]
    _common(d, 2, 3)
    assert d["dtype"] == "f32" and d["config"]["poses"] == 3000 and d["config"]["iters"] == 300
    r = d["roofline"]
    assert r["bound"] in ("alu", "hbm", "tensor") and r["unit"] == "TFLOP/s"
    assert 0 < r["achieved"] < r["peak"] and abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-9
    assert r["kernel_ms_avg"] <= d["ms_per_step"] * 1.001
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert d["clocks"]["sm_mhz"] > 0 and isinstance(d["clocks"]["reasons"], list)
    assert d["gpu_launches"] >= 2 * 1  # one LS launch (+ best-of-run) per timed step
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] > 0 and cb["sample"]
    # north_star's accuracy report on the same workload: sane relaxed poses inside the bounds
    rel = d["parity"]["relaxed_poses"]
    assert rel["n_sane_poses"] > 0 and rel["sane_max_abs_dE"] <= 1e-3 and rel["sane_max_grad_rel_err"] <= 1e-4
