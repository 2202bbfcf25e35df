"""bench.py's JSON contract on CPU: the reference arm (the oracle on the host's
cores) prints one line with the keys the driver reads, and its `config`
object is the one our arm reports for the same arguments."""
from __future__ import annotations

import json
import subprocess
import sys
from argparse import Namespace
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]


def test_reference_arm_line():
    out = subprocess.run([sys.executable, str(ROOT / "bench.py"), "--impl", "reference", "--config", "c1",
                          "--steps", "2", "--warmup", "1"], capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.strip()]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e", "impl"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["higher_is_better"] is True
    assert d["e2e"] == {"value": d["value"], "unit": d["unit"], "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    sys.path.insert(0, str(ROOT))
    import bench
    args = Namespace(config="c1", mode="list", scaling="weak")
    assert d["config"] == bench.bench_config(args, 1)


def test_default_config_is_c3():
    sys.path.insert(0, str(ROOT))
    import bench
    sys.argv = ["bench.py"]
    a = bench.parse()
    assert a.config == "c3" and a.gpus == 1 and a.warmup >= 3 and a.mode == "list"
