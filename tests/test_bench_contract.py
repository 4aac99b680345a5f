"""bench.py keeps the driver's JSON-line contract (one line on stdout, the keys the driver and
the judge read).  The reference arm (the CPU oracle, tier framing) runs anywhere; the product arm
needs the GPU."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BASE_KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
             "scaling", "vs_baseline", "dtype", "data", "config", "e2e"}


def _run(args, timeout):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], cwd=ROOT,
                       capture_output=True, text=True, timeout=timeout)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.strip()]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


def test_reference_arm_json_line():
    d = _run(["--impl", "reference", "--config", "grid256", "--steps", "1", "--warmup", "1"], 300)
    assert BASE_KEYS <= d.keys()
    assert d["impl"] == "reference" and d["unit"] == "GTEPS" and d["value"] > 0
    assert d["config"]["workload"] == "grid256"
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["value"] == d["value"] and d["e2e"]["h2d_bytes_per_step"] == 0


@pytest.mark.gpu
def test_product_arm_json_line():
    d = _run(["--config", "grid256", "--steps", "3", "--warmup", "3", "--cpu-seconds", "1"], 900)
    assert BASE_KEYS <= d.keys()
    assert d["unit"] == "GTEPS" and d["value"] > 0 and d["higher_is_better"] is True
    assert d["gpu_launches"] > 0
    r = d["roofline"]
    assert {"bound", "achieved", "peak", "unit", "frac", "traffic"} <= r.keys() and r["bound"] == "hbm"
    assert abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-3
    c = d["cpu_baseline"]
    assert {"value", "unit", "cores", "kind", "sample"} <= c.keys() and c["kind"] == "oracle"
    e = d["e2e"]
    assert {"value", "unit", "h2d_bytes_per_step", "d2h_bytes_per_step"} <= e.keys()
    assert e["d2h_bytes_per_step"] >= 4 * d["config"]["n"]          # the parent array comes back
    assert {"sm_mhz", "sm_max_mhz", "reasons"} <= d["clocks"].keys()
    assert d["validation"] and all(v["i6"] == 1 for v in d["validation"].values())
    sp = d["span"]["roots"][0]                                       # headline root 0 of the grid
    assert sp["root"] == 0 and sp["bfs_ecc"] == 255 + 255 and 0 < sp["frac_of_floor"] <= 1


def test_gpus_flag_relaunches_under_torchrun():
    """`bench.py --gpus 2` without torchrun re-launches itself with 2 ranks (torch.distributed.run);
    the reference arm runs on rank 0 only, the other rank exits 0 without work: one JSON line."""
    d = _run(["--impl", "reference", "--gpus", "2", "--config", "grid256", "--steps", "1", "--warmup", "0"], 600)
    assert d["impl"] == "reference" and d["n_gpus"] == 2 and d["value"] > 0
