"""Host-side checks of bench.py (no GPU): the byte model, the clocks parser and
the reference arm (the oracle on the host cores)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def test_gather_bytes_model():
    # GCN: per edge 4F + 4 (colidx) + 4 (coef); per row 4F (Y) + 8 (rowptr)
    assert bench.gather_bytes("gcn", 2, 10, 3) == 10 * (12 + 8) + 2 * (12 + 8)
    # GIN: per edge 4F + 4; per row self + Y + rowptr
    assert bench.gather_bytes("gin", 2, 10, 3) == 10 * (12 + 4) + 2 * (24 + 8)
    # GAT: per edge 4F + 4 + 4 (el); per row Y + rowptr + er
    assert bench.gather_bytes("gat", 2, 10, 3) == 10 * (12 + 8) + 2 * (12 + 12)
    assert bench.gather_bytes("gcn2", 2, 10, 3) == 2 * bench.gather_bytes("gcn", 2, 10, 3)
    # Reddit GCN matches SURVEY 8(d): 277.5 GB per call
    assert abs(bench.gather_bytes("gcn", 232965, 114615892, 602) / 1e9 - 277.5) < 0.1


def test_clock_sampler_summary():
    c = bench.ClockSampler(0, period_ms=0)
    c.lines = ["0, 1900, 1965, 800.1, 0x4, Not Active, Not Active, Not Active, Active",
               "0, 1700, 1965, 990.0, 0x4, Not Active, Not Active, Not Active, Active",
               "0, 1800, 1965, 950.0, 0x0, Not Active, Not Active, Not Active, Not Active",
               "garbage"]
    s = c.summary()
    assert s["sm_mhz"] == 1800 and s["sm_max_mhz"] == 1965
    assert s["reasons"] == ["sw_power_cap"] and s["samples"] == 3


def test_peak_from_measured_file():
    v, src = bench.peak_hbm()
    assert v > 1000
    assert ("measured" in src) == os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json"))


@pytest.mark.slow
def test_reference_arm_runs_on_host():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                        "--workload", "cora", "--steps", "1", "--warmup", "1"],
                       capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    d = json.loads(r.stdout.strip().splitlines()[-1])
    assert d["impl"] == "reference" and d["value"] > 0 and d["gpu_launches"] == 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["e2e"]["h2d_bytes_per_step"] == 0


def test_l2_gather_peak_parses_committed_probe():
    """bench.py's L2 roofline reads the committed probe: the 256-byte-row,
    L2-resident (< 80 MB table) entry with the highest bandwidth."""
    import bench
    p = bench.l2_gather_peak()
    assert p is not None
    assert p["row_bytes"] == 256 and p["table_MB"] < 80
    assert 5000 < p["GBs"] < 40000
