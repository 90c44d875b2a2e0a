"""Mutation check of the oracle pins: each mutation plants a plausible mistake
in a scratch copy of oracle/tlp_oracle.c (a dropped factor, a wrong sign or
index, a loosened bound term), rebuilds it there and runs the CPU pin suites
against it.  Every mutation must be caught (at least one failing test).

usage: python scripts/oracle_mutations.py   (CPU only, ~2 min)
"""
import os
import shutil
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# (name, original snippet, mutated snippet, occurrence index)
MUTATIONS = [
    ("gat bound drops alpha", "a += alpha[e - e0] * fabs(x);", "a += fabs(x);", 0),
    ("gat_mh bound drops alpha", "a += alpha[e - e0] * fabs(x);", "a += fabs(x);", 1),
    ("gin bound self x10", "double s = self, a = fabs(self);", "double s = self, a = 10.0 * fabs(self);", 0),
    ("gin self drops eps", "double self_w = 1.0 + eps;", "double self_w = 1.0;", 0),
    ("gcn bound drops c_in", "A[i * F + f] = c_in * a;", "A[i * F + f] = a;", 0),
    ("gcn bound drops c_out", "a += fabs(term);\n            }\n            Y[i * F + f] = c_in * s;",
     "a += fabs(w * (double)X[u * ldx + f]);\n            }\n            Y[i * F + f] = c_in * s;", 0),
    ("gcn both uses in-degree for c_out", "int32_t od = out_deg[u];", "int32_t od = (int32_t)(rowptr[u + 1] - rowptr[u]);", 0),
    ("sage bound drops 1/count", "A[i * F + f] = inv * a;", "A[i * F + f] = a;", 0),
    ("sage self not in the count", "int64_t cnt = d + (include_self ? 1 : 0);", "int64_t cnt = d;", 0),
    ("leaky relu sign", "return x >= 0.0 ? x : slope * x;", "return x >= 0.0 ? x : -slope * x;", 0),
    ("gat softmax max omitted from z", "z += exp(alpha[k] - m);", "z += exp(alpha[k]);", 0),
    ("gat er index without row_offset", "double er_v = (double)er[row_offset + v];", "double er_v = (double)er[v];", 0),
    ("gin self row without row_offset", "double self = self_w * (double)X[(row_offset + v) * ldx + f];", "double self = self_w * (double)X[v * ldx + f];", 0),
    ("sage self row without row_offset", "double x = (double)X[(row_offset + v) * ldx + f];", "double x = (double)X[v * ldx + f];", 0),
    ("gcn backward bound transposed", "A[u * F + f] += fabs(term);", "A[u * F + f] += fabs(coef);", 0),
    ("gin backward bound eps", "A[u * F + f] = fabs(t);", "A[u * F + f] = fabs((double)dY[u * lddy + f]);", 0),
    ("gat backward bound drops SA", "double bt = fabs(lr) * a * (G[e - e0] + SA);", "double bt = fabs(lr) * a * G[e - e0];", 0),
    ("gat backward bound slope", "double bt = fabs(lr) * a * (G[e - e0] + SA);", "double bt = a * (G[e - e0] + SA);", 0),
    ("gat backward dX bound", "AdX[u * F + f] += fabs(term);", "AdX[u * F + f] += fabs((double)dY[v * lddy + f]);", 0),
    ("epilogue bound ignores bias", "A[i * F + f] += fabs((double)bias[f]);", "A[i * F + f] += 0.0;", 0),
    ("project bound", "b += fabs(t);", "b += t;", 0),
    ("partition floor off by one", "while (r < n && rowptr[r] < target)", "while (r < n && rowptr[r] <= target)", 0),
    ("out-degree index", "out_deg[colidx[e]] += 1;", "out_deg[colidx[e] % (n_src > 1 ? n_src - 1 : 1)] += 1;", 0),
]

SUITES = ["tests/test_oracle_pins.py", "tests/test_oracle_bounds.py"]


def replace_nth(s, old, new, k):
    i = -1
    for _ in range(k + 1):
        i = s.find(old, i + 1)
        if i < 0:
            raise SystemExit("snippet not found: %r (occurrence %d)" % (old, k))
    return s[:i] + new + s[i + len(old):]


def main():
    src = open(os.path.join(ROOT, "oracle", "tlp_oracle.c")).read()
    survivors = []
    for name, old, new, k in MUTATIONS:
        with tempfile.TemporaryDirectory() as d:
            for sub in ("oracle", "synth", "tests"):
                shutil.copytree(os.path.join(ROOT, sub), os.path.join(d, sub),
                                ignore=shutil.ignore_patterns("*.so", "__pycache__"))
            shutil.copy(os.path.join(ROOT, "pytest.ini"), d)
            with open(os.path.join(d, "oracle", "tlp_oracle.c"), "w") as f:
                f.write(replace_nth(src, old, new, k))
            r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider"]
                               + SUITES, cwd=d, capture_output=True, text=True)
            caught = r.returncode != 0
            last = (r.stdout.strip().splitlines() or [""])[-1]
            print("%-40s %s  (%s)" % (name, "caught" if caught else "SURVIVED", last), flush=True)
            if not caught:
                survivors.append(name)
    print("%d/%d mutations caught" % (len(MUTATIONS) - len(survivors), len(MUTATIONS)))
    return 1 if survivors else 0


if __name__ == "__main__":
    sys.exit(main())
