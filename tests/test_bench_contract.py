"""bench.py's contract pieces that run without a GPU: the reference arm (the
oracle on host cores, per the tier rules) prints one well-formed JSON line,
and the workload / config helpers match BASELINE.json's configs."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def test_models():
    assert bench.flops_per_matrix(3) == 9.0
    assert bench.bytes_per_matrix(32) == 4228
    a = type("A", (), dict(workload="c2", n=None, batch=None, chunk=None, kind=None, gpus=1))()
    w = bench.workload(a)
    assert (w["n"], w["batch"], w["chunk"]) == (16, 1 << 20, 32)
    a.workload = "c4n48"
    assert bench.workload(a)["n"] == 48
    a.workload = "c5"
    w = bench.workload(a)
    assert w["global_batch"] and w["batch"] == 1 << 25 and w["fail_period"] == 1009
    cfg = bench.config_of(bench.workload(type("A", (), dict(workload="c1", n=None, batch=None,
                                                           chunk=None, kind=None, gpus=1))()), a)
    assert "flushed" in cfg["l2"]


def test_reference_arm_json_line():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                          "--n", "6", "--batch", "2000", "--steps", "2", "--warmup", "1"],
                         capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert out.returncode == 0, out.stderr
    lines = [l for l in out.stdout.splitlines() if l.strip()]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
              "higher_is_better", "scaling", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["unit"] == "Gflop/s"
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["metric"] == json.load(open(os.path.join(ROOT, "BASELINE.json")))["metric"]


def test_reference_arm_nonzero_rank_exits_quietly():
    env = dict(os.environ, RANK="1", WORLD_SIZE="2")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                          "--n", "4", "--batch", "100", "--steps", "1", "--warmup", "0"],
                         capture_output=True, text=True, timeout=300, cwd=ROOT, env=env)
    assert out.returncode == 0 and out.stdout.strip() == ""


def test_default_workload_is_headline_config(monkeypatch):
    """No flags -> BASELINE configs[2] (n=32, 4M, ALS, chunk 32): the largest
    single-GPU config, the one the driver's bench line is quoted on."""
    monkeypatch.setattr(sys, "argv", ["bench.py"])
    a = bench.parse()
    w = bench.workload(a)
    assert (w["n"], w["batch"], w["chunk"], w["kind"]) == (32, 1 << 22, 32, "als")
    assert "configs[2]" in w["desc"]
    cfgs = json.load(open(os.path.join(ROOT, "BASELINE.json")))["configs"]
    assert "n=32, batch=4M" in cfgs[2]
    assert bench.parse_ns(a.per_n) == list(range(1, 65))
    assert bench.parse_ns("1-3,8,16-17") == [1, 2, 3, 8, 16, 17]


def test_host_budget_is_capped():
    b = bench.host_budget_bytes(8)
    assert 0 < b <= 48 << 30
    assert bench.host_budget_bytes(1) >= b
