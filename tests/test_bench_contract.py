"""The driver's bench contract on the CPU: `bench.py --impl reference` (the oracle as the reference
arm, runnable without a GPU) prints exactly one JSON line with the keys the driver reads."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "3",
                          "--warmup", "1", "--size", "1024"], cwd=ROOT, capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.strip()]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference"
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "higher_is_better", "dtype", "data", "config",
              "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["value"] > 0 and d["steps"] == 3 and d["warmup"] == 1 and d["higher_is_better"] is True
    assert d["config"]["workload"].startswith("C2: 2D 5-point Jacobi 1024x1024 fp32")
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["unit"] == d["unit"]
    assert "3 sweeps" in d["cpu_baseline"]["sample"]


import pytest  # noqa: E402


@pytest.mark.gpu
def test_accmg_arm_json_line():
    """The accmg arm at a small field: one JSON line with roofline, e2e, clocks, launches."""
    from tests.gpu_util import need_gpu
    need_gpu()
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--size", "4096", "--steps", "5",
                          "--warmup", "3", "--e2e-steps", "1", "--e2e-sweeps", "4"], cwd=ROOT, capture_output=True,
                         text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.strip()]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "clocks", "e2e", "gpu_launches", "cpu_baseline"):
        assert k in d, k
    assert d["steps"] == 5 and d["warmup"] == 3 and d["gpu_launches"] >= 5
    r = d["roofline"]
    assert r["bound"] == "hbm" and r["unit"] == "GB/s" and 0 < r["frac"] < 1.1 and r["peak"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert "sm_mhz" in d["clocks"] and "reasons" in d["clocks"]


def test_self_launch_command(monkeypatch):
    """`python bench.py --gpus N` without torchrun re-runs itself as N ranks through
    torch.distributed.run on 127.0.0.1 (the driver may call it either way)."""
    sys.path.insert(0, ROOT)
    import bench
    seen = {}

    def fake_call(cmd, **kw):
        seen["cmd"] = cmd
        return 0

    monkeypatch.setattr(bench.subprocess, "call", fake_call)
    monkeypatch.delenv("WORLD_SIZE", raising=False)
    monkeypatch.setattr(sys, "argv", ["bench.py", "--gpus", "4", "--steps", "7", "--warmup", "3"])
    try:
        bench.main()
    except SystemExit as e:
        assert e.code == 0
    cmd = seen["cmd"]
    assert cmd[1:3] == ["-m", "torch.distributed.run"]
    assert "--nproc-per-node=4" in cmd and "127.0.0.1" in cmd
    assert cmd[-6:] == ["--gpus", "4", "--steps", "7", "--warmup", "3"]
    assert cmd[cmd.index("--master-addr") + 1] == "127.0.0.1"


@pytest.mark.gpu
def test_accmg_arm_two_ranks_self_launched():
    """`python bench.py --gpus 2` with no torchrun around it: two ranks (sharing the GPU on a
    one-GPU box, one per GPU otherwise), one JSON line from rank 0 with n_gpus = 2."""
    from tests.gpu_util import need_gpu
    need_gpu()
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--size", "4096", "--steps",
                          "5", "--warmup", "3", "--e2e-steps", "1", "--e2e-sweeps", "4"], cwd=ROOT, capture_output=True,
                         text=True, timeout=900, env=env)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.strip().startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["config"]["partitions"] == 2
    assert d["inter_gpu_bytes_per_loop"] > 0 and "e2e" in d
