"""Host-side logic of bench.py (CPU): the run sizing shared by both arms and the
reference arm's JSON line (the oracle on a bounded C3 sample)."""
import json
import os
import subprocess
import sys
import types

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402

GiB = 1 << 30


def _args(**kw):
    d = dict(block=2 << 20, budget_gib=170.0, oversub=1.5)
    d.update(kw)
    return types.SimpleNamespace(**d)


def test_plan_sizes_clamps_and_reports(monkeypatch):
    monkeypatch.setattr(bench, "_mem_available", lambda: None)
    b, a, pool, why = bench.plan_sizes(_args(), 180 * GiB, 1)
    assert (b, why) == (170 * GiB, None) and a == int(b * 1.5) // (2 << 20) * (2 << 20)
    assert pool == a - b + 2 * GiB
    b, _, _, why = bench.plan_sizes(_args(), 100 * GiB, 1)
    assert b == 95 * GiB and why == "free HBM"
    monkeypatch.setattr(bench, "_mem_available", lambda: 200 * GiB)
    b, a, pool, why = bench.plan_sizes(_args(), 180 * GiB, 8)      # 8 ranks share host RAM
    assert "host RAM" in why and pool <= 0.85 * 200 * GiB / 8 + 1
    assert b % (2 << 20) == 0


def test_reference_arm_line():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                          "--warmup", "1", "--budget-gib", "2"], capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    line = json.loads(out.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["unit"] == "iter/s" and line["value"] > 0
    assert line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["cores"] == 1
    assert line["e2e"]["h2d_bytes_per_step"] == 0 and line["config"]["budget_bytes"] == 2 * GiB
