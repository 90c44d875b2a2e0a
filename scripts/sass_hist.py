"""Per-SASS-instruction execution counts of an ncu source page (--page source
--csv --print-source sass), grouped by execution count: shows how many
instructions run once per work item, once per gather step, etc., and where
the warp-stall samples fall.  usage: python scripts/sass_hist.py <sass.csv>..."""
import collections
import csv
import sys


def num(x):
    x = x.replace(",", "")
    try:
        return float(x)
    except ValueError:
        return 0.0


for f in sys.argv[1:]:
    rows = list(csv.reader(open(f)))
    hdr = rows[1]
    data = [dict(zip(hdr, r)) for r in rows[2:] if len(r) == len(hdr)]
    tot_i = sum(num(d["Instructions Executed"]) for d in data)
    tot_s = sum(num(d["Warp Stall Sampling (All Samples)"]) for d in data)
    c, n, smp = collections.Counter(), collections.Counter(), collections.Counter()
    for d in data:
        k = int(num(d["Instructions Executed"]))
        c[k] += k
        n[k] += 1
        smp[k] += num(d["Warp Stall Sampling (All Samples)"])
    print(f"== {f}: {rows[0][1]}")
    print(f"   warp instructions {tot_i:.0f}, stall samples {tot_s:.0f}")
    for k, v in sorted(c.items(), key=lambda kv: -kv[1])[:8]:
        print(f"   executed {k:>8d} times: {n[k]:4d} SASS instructions, {v / tot_i:6.1%} of instructions, "
              f"{smp[k] / max(tot_s, 1):6.1%} of stall samples")
