"""CPU-side checks of the C-ABI library: it loads, exports every symbol that
include/tlp.h declares, and its pure host functions are bit-exact against the
oracle (no compute calls: there is no GPU here)."""
import os
import re

import numpy as np
import pytest

import oracle
import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    names = set()
    for fn in os.listdir(os.path.join(ROOT, "include")):
        if fn.endswith(".h"):
            src = open(os.path.join(ROOT, "include", fn)).read()
            src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
            names |= set(re.findall(r"\b(tlp_[a-z_]+)\s*\(", src))
    return names


def test_library_exports_every_declared_symbol():
    import ctypes
    import paper_conf_hpdc_fujh22_b200 as tlp
    declared = _declared()
    assert len(declared) >= 20
    lib = ctypes.CDLL(tlp.LIB_PATH)
    for name in declared:
        assert hasattr(lib, name), name
    # and the binding wraps every one of them under the same name
    assert declared == set(tlp.C_SYMBOLS), declared ^ set(tlp.C_SYMBOLS)


def test_version_and_status_strings():
    import paper_conf_hpdc_fujh22_b200 as tlp
    assert tlp.tlp_version() == 1
    assert tlp.tlp_status_string(0) == "TLP_OK"
    assert tlp.tlp_status_string(2) == "TLP_ERR_INVALID_GRAPH"


def test_library_is_sm100a_only():
    """The cubin inside libtlp.so targets sm_100a (no PTX JIT fallback)."""
    import shutil
    import subprocess
    import paper_conf_hpdc_fujh22_b200 as tlp
    cuobjdump = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(cuobjdump):
        pytest.skip("cuobjdump not available")
    out = subprocess.run([cuobjdump, "--list-elf", tlp.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    archs = set(re.findall(r"sm_(\d+a?)", out))
    assert archs == {"100a"}, archs


def test_sass_cache_policy_descriptors_are_register_pairs():
    """Every memory instruction that carries an L2 cache-policy descriptor
    (desc[URx], a 64-bit uniform-register pair) names an even register.
    ptxas 12.9 emitted LDGSTS with desc[UR1] in the cp.async kernels once they
    also held the Cluster Launch Control scheduler (an illegal instruction at
    run time); this guards the built library against that miscompile."""
    import shutil
    import subprocess
    import paper_conf_hpdc_fujh22_b200 as tlp
    cuobjdump = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(cuobjdump):
        pytest.skip("cuobjdump not available")
    sass = subprocess.run([cuobjdump, "-sass", tlp.LIB_PATH], capture_output=True, text=True).stdout
    regs = [int(r) for r in re.findall(r"desc\[UR(\d+)\]", sass)]
    assert regs, "no cache-policy descriptors found (disassembly failed?)"
    odd = sorted({r for r in regs if r % 2})
    assert not odd, f"odd uniform registers used as descriptors: {odd}"
    assert "UGETNEXTWORKID" in sass  # the CLC scheduler is compiled in


@pytest.mark.parametrize("parts", [1, 2, 3, 4, 7, 8])
def test_partition_rows_bit_exact(parts):
    import paper_conf_hpdc_fujh22_b200 as tlp
    for name in ("cora", "pubmed"):
        rp, _ = synth.dataset_graph(name, device="cpu")
        assert tlp.tlp_partition_rows(rp, parts).tolist() == oracle.partition(rp, parts).tolist()
    for seed in range(5):
        rp, _ = synth.random_graph(50, 50, 300, seed, isolated_tail=seed * 3)
        assert tlp.tlp_partition_rows(rp, parts).tolist() == oracle.partition(rp, parts).tolist()
    # a hub holding more than E/P edges gives empty partitions; b_P = N
    rp = np.array([0, 100, 101, 102, 102, 102], np.int64)
    assert tlp.tlp_partition_rows(rp, parts).tolist() == oracle.partition(rp, parts).tolist()
    rp0 = np.zeros(6, np.int64)
    assert tlp.tlp_partition_rows(rp0, parts).tolist() == oracle.partition(rp0, parts).tolist()


def test_partition_rows_rejects_bad_input():
    import paper_conf_hpdc_fujh22_b200 as tlp
    with pytest.raises(tlp.TlpError):
        tlp.tlp_partition_rows(np.array([1, 2, 3], np.int64), 2)
    with pytest.raises(tlp.TlpError):
        tlp.tlp_partition_rows(np.array([0, 2, 3], np.int64), 0)


def test_no_cpu_fallback_for_features():
    import torch
    import paper_conf_hpdc_fujh22_b200 as tlp
    with pytest.raises(TypeError):
        tlp._feat(torch.zeros(4, 3), None)
    with pytest.raises(TypeError):
        tlp._vec_cuda(torch.zeros(4), "el")


def test_missing_library_fails_loudly(tmp_path):
    """Without libtlp.so the package does not import (no silent fallback)."""
    import subprocess
    import sys
    env = dict(os.environ, TLP_LIB_PATH=str(tmp_path / "absent" / "libtlp.so"))
    r = subprocess.run([sys.executable, "-c", "import paper_conf_hpdc_fujh22_b200"], cwd=ROOT,
                       env=env, capture_output=True, text=True, timeout=300)
    assert r.returncode != 0
    assert "ImportError" in r.stderr


def test_product_package_does_not_import_oracle():
    """The product path never touches oracle/ (and vice versa)."""
    pkg = os.path.join(ROOT, "paper_conf_hpdc_fujh22_b200")
    bad = re.compile(r"^\s*(import oracle|from oracle|.*liboracle|.*tlp_oracle)", re.M)
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".h", ".cpp")):
                assert not bad.search(open(os.path.join(dirpath, f)).read()), f
    bad2 = re.compile(r"^\s*(import paper_conf|from paper_conf|#include .tlp)", re.M)
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c")):
            assert not bad2.search(open(os.path.join(ROOT, "oracle", f)).read()), f
