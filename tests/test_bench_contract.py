"""bench.py output contract: one JSON line with the keys the driver reads.
The reference arm (the CPU oracle) runs here without a GPU; the GPU arm is
checked under -m gpu with a short run."""
import json
import subprocess
import sys
from pathlib import Path

import pytest

ROOT = Path(__file__).resolve().parent.parent


def _run(args, timeout):
    out = subprocess.run([sys.executable, str(ROOT / "bench.py"), *args], capture_output=True, text=True,
                         timeout=timeout, cwd=str(ROOT))
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.strip()]
    assert len(lines) == 1, out.stdout
    return json.loads(lines[0])


def test_reference_arm_contract():
    d = _run(["--impl", "reference", "--steps", "2", "--warmup", "3"], timeout=600)
    base = json.loads((ROOT / "BASELINE.json").read_text())
    assert d["impl"] == "reference" and d["metric"] == base["metric"]
    assert d["unit"] == "samples/s" and d["higher_is_better"] is True and d["value"] > 0
    assert d["warmup"] >= 3 and d["steps"] == 2
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] == d["value"] and cb["sample"]
    assert d["e2e"] == {"value": d["value"], "unit": d["unit"], "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}


@pytest.mark.gpu
def test_gpu_arm_contract():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    d = _run(["--steps", "5", "--warmup", "3", "--secondary", "none", "--e2e-steps", "1", "--cpu-seconds", "1"],
             timeout=900)
    base = json.loads((ROOT / "BASELINE.json").read_text())
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e", "gpu_launches", "clocks"):
        assert k in d, k
    assert d["metric"] == base["metric"] and d["n_gpus"] == 1 and d["scaling"] == "weak"
    assert d["vs_baseline"] is None and d["data"] == "synthetic" and "workload" in d["config"]
    r = d["roofline"]
    assert r["bound"] == "hbm" and r["unit"] == "GB/s" and 0 < r["frac"] < 1.2
    assert abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-9
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert d["gpu_launches"] == 2 * d["steps"]
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    # round-2 reporting (VERDICT r1 missing 5): nominal-peak fraction, per-rank H2D and overlap,
    # placement, format statistics, value = mode A / e2e = mode B labels
    assert abs(r["frac_nominal_8tbs"] - r["achieved"] / 8000.0) < 1e-9
    assert len(d["per_rank"]) == 1 and d["per_rank"][0]["h2d_gbs"] > 0 and 0 < d["per_rank"][0]["overlap"] <= 1.5
    assert len(d["config"]["placement"]) == 1 and "mode A" in d["config"]["workload"]
    st = d["config"]["stream_stats"]
    assert st["nU_mean"] > 0 and st["G_slab0_mean"] > 0 and st["kw_slab0"]


@pytest.mark.gpu
@pytest.mark.parametrize("scaling", ["weak", "strong"])
def test_gpu_arm_two_ranks(scaling):
    """The multi-rank path of bench.py (torchrun, one process per rank, barrier +
    MAX over ranks, whole-job throughput) for BOTH workloads (C2 headline + C4
    secondary), with two ranks sharing this GPU over gloo (the driver's scaling
    run uses NCCL, one GPU per rank)."""
    import os
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    env = dict(os.environ, SPP_DIST_BACKEND="gloo")
    port = 29731 + (scaling == "strong")
    out = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
                          "--master-addr=127.0.0.1", f"--master-port={port}", str(ROOT / "bench.py"), "--gpus", "2",
                          "--batch", "32", "--secondary-batch", "4", "--pool", "2", "--steps", "3", "--warmup", "3",
                          "--e2e-steps", "1", "--scaling", scaling],
                         capture_output=True, text=True, timeout=1200, cwd=str(ROOT), env=env)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.strip().startswith("{")]
    assert len(lines) == 1, out.stdout
    d = json.loads(lines[0])
    total = 64 if scaling == "weak" else 32
    assert d["n_gpus"] == 2 and d["scaling"] == scaling and d["value"] > 0 and d["cpu_baseline"] is None
    assert d["config"]["samples_per_step_all_ranks"] == total
    assert d["value"] == pytest.approx(total * 3 / (d["ms_per_step"] * 3 / 1e3), rel=1e-6)
    assert d["e2e"]["value"] > 0 and d["gpu_launches"] == 2 * 3
    assert len(d["per_rank"]) == 2 and all(r["h2d_gbs"] > 0 and r["overlap"] > 0 for r in d["per_rank"])
    assert len(d["config"]["placement"]) == 2
    s = d["secondary"]                          # DeepCAM C4 at N = 2 as well
    assert s["cfg"] == "C4" and s["value"] > 0 and s["units_per_step"] == (8 if scaling == "weak" else 4)
    assert s["roofline"]["frac"] > 0 and len(s["per_rank"]) == 2 and s["cpu_baseline"] is None
