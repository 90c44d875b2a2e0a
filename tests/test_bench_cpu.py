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


def test_l2_ceiling_probe_builds_and_exports():
    """The in-run L2 gather-ceiling probe (bench_probe/l2_ceiling.cu) is built
    by build() and exports its C entry point (it runs only on a GPU)."""
    import ctypes
    p = os.path.join(ROOT, "bench_probe", "libl2c.so")
    if not os.path.exists(p):
        sys.path.insert(0, os.path.join(ROOT, "paper_conf_hpdc_fujh22_b200"))
        import _build
        _build.build_probe()
    lib = ctypes.CDLL(p)
    assert hasattr(lib, "l2c_run")


def test_launcher_two_ranks_gloo():
    """`bench.py --gpus 2` without a launcher starts two ranks itself
    (torch.distributed.run over 127.0.0.1); the self-test rank body runs on CPU
    with gloo: libtlp's host partition equals the oracle's rule on every rank,
    max/sum reductions over ranks, rank 0 prints one JSON line."""
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--selftest"],
                       capture_output=True, text=True, timeout=300, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.strip().splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["bounds_match_oracle"] and d["edges_total"] == d["nnz"]
    assert d["edges_max_rank"] <= d["nnz"] // 2 + 200


def test_gpus_mismatch_with_world_size_is_an_error():
    env = dict(os.environ, WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "4", "--selftest"],
                       capture_output=True, text=True, timeout=120, cwd=ROOT, env=env)
    assert r.returncode == 2 and "WORLD_SIZE" in r.stderr
