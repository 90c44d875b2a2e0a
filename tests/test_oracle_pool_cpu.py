"""CPU checks of the process-pool parity driver (tests/oracle_pool.py): it
reproduces the single-process oracle comparison and flags a single bad
element, a NaN and a wrong row."""
import numpy as np

import oracle
import synth
from oracle_pool import check_rows


def _graph():
    rp, ci = synth.chung_lu(3000, 90000, 0.5, 3, device="cpu")
    X = synth.features(3000, 37, 40, seed=2)
    return rp, ci, X


def test_pool_passes_oracle_output_and_flags_errors():
    rp, ci, X = _graph()
    Y, _ = oracle.gcn(rp, ci, X, "both", F=37)
    Yg = np.zeros((3000, 40), np.float32)
    Yg[:, :37] = Y.astype(np.float32)
    r = check_rows("gcn", rp, ci, X, Yg, procs=4, F=37, norm="both")
    assert r["rows"] == 3000 and r["bad"] == 0 and r["worst"] < 0.2
    Yb = Yg.copy()
    Yb[1234, 5] += 1e-2
    Yb[17, 36] = np.nan
    r = check_rows("gcn", rp, ci, X, Yb, procs=4, F=37, norm="both")
    assert r["bad"] == 2
    # a different op's output fails
    r = check_rows("gin", rp, ci, X, Yg, procs=4, F=37, eps=0.1)
    assert r["bad"] > 0


def test_pool_gat_and_row_subset():
    rp, ci, X = _graph()
    el, er = synth.normal(3000, 1), synth.normal(3000, 2)
    rows = np.array([0, 5, 77, 2999])
    Y, _ = oracle.gat(rp, ci, X, el, er, 0.2, F=37)
    r = check_rows("gat", rp, ci, X, Y.astype(np.float32), rows=rows, procs=2, el=el, er=er,
                   F=37, slope=0.2)
    assert r["rows"] == 4 and r["bad"] == 0
