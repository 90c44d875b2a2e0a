"""Summarise a round's gpurun_out/<round> evidence into profiles/ (tracked)."""
import csv, json, os, subprocess, sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "scripts"))
from ncu_summary import summarise  # noqa: E402

R = sys.argv[1] if len(sys.argv) > 1 else "r01"
src = os.path.join(ROOT, "gpurun_out", R)
dst = os.environ.get("PROFILES_OUT") or os.path.join(ROOT, "profiles")
os.makedirs(dst, exist_ok=True)
out = [f"# Round {R} profile summary\n"]

# bench line
bj = os.path.join(src, "bench.json")
bench = None
if os.path.exists(bj):
    bench = json.load(open(bj))
    json.dump(bench, open(os.path.join(dst, f"{R}_bench.json"), "w"), indent=1)
    out.append("## bench.py (default: Reddit-shaped GCN+GIN+GAT step)\n")
    out.append(f"value {bench['value']} GB/s gather-model, ms/step {bench['ms_per_step']}, clocks {bench['clocks']}\n")
    for op, d in bench["ops"].items():
        out.append(f"* {op}: {d['ms_mean']} ms mean, {d['gather_GBs']} GB/s gather-model ({d['frac_of_8TBs']} of 8 TB/s)\n")
    out.append("\n")

# bench lines of the other workloads
import glob
extra = sorted(glob.glob(os.path.join(src, "bench_*.json")))
if extra:
    out.append("## other workloads (bench.py --workload W, one line each)\n\n")
    out.append("| workload | ms/step | per op ms (mean) | GB/s gather-model | e2e GB/s | sm MHz |\n|---|---|---|---|---|---|\n")
    for f in extra:
        try:
            b = json.loads(open(f).read().strip().splitlines()[-1])
        except Exception:
            continue
        wl = os.path.basename(f)[6:-5]
        json.dump(b, open(os.path.join(dst, f"{R}_bench_{wl}.json"), "w"), indent=1)
        ops = ", ".join(f"{k} {v['ms_mean']}" for k, v in b.get("ops", {}).items())
        e2e = (b.get("e2e") or {}).get("value")
        out.append(f"| {wl} | {b['ms_per_step']} | {ops} | {b['value']} | {e2e} | {b['clocks']['sm_mhz']} |\n")
        if b.get("paper_context"):
            out.append(f"| ↳ paper V100 (F=32) | | {b['paper_context']['v100_ms']} | B200/V100 {b['paper_context']['b200_over_v100']} | | |\n")
    out.append("\n")

# launch list: share of each kernel in the step
lc = os.path.join(src, "launches.csv")
if os.path.exists(lc):
    rows = list(csv.reader(open(lc)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[start]
    ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
    tot, cnt = defaultdict(float), defaultdict(int)
    for r in rows[start + 1:]:
        if len(r) > vi:
            tot[r[ki]] += float(r[vi].replace(",", ""))
            cnt[r[ki]] += 1
    agg = {k: v for k, v in tot.items() if "k_agg" in k or "k_prescale" in k or "k_gat_alpha" in k}
    T = sum(agg.values())
    out.append("## ncu launch list (gpu__time_duration.sum, --clock-control none; cold, serialised)\n")
    out.append("Share of the aggregation kernels within the timed bench step (2 steps):\n\n")
    for k, v in sorted(agg.items(), key=lambda x: -x[1]):
        out.append(f"* {k}: {v / 1e6 / cnt[k]:.2f} ms per launch, {cnt[k]} launches, {100 * v / T:.1f}% of the step's kernel time\n")
    out.append("\n(other launches in the file are the one-time synthetic-graph generation and graph create)\n\n")
    with open(os.path.join(dst, f"{R}_launches.csv"), "w") as f:
        f.write(open(lc).read())

# ncu --set full reports
traffic = {}
names = {"reddit_gcn": ("reddit", "gcn"), "reddit_gin": ("reddit", "gin"),
         "reddit_gat": ("reddit", "gat"), "reddit_gat_alpha": ("reddit", "gat_alpha"),
         "products_gat": ("products", "gat"),
         "reddit_gatb": ("reddit_gat_bwd", "gat_bwd")}
out.append("## ncu --set full (one launch each, --clock-control none, cold L2)\n\n")
for nm, (wl, op) in names.items():
    p = os.path.join(src, nm + ".ncu-rep")
    if not os.path.exists(p):
        continue
    for d in summarise(p):
        k = d.pop("kernel")
        rd = float(d["dram_rd"][0]) * (1e9 if d["dram_rd"][1].startswith("G") else 1e6)
        wr = float(d["dram_wr"][0]) * (1e9 if d["dram_wr"][1].startswith("G") else 1e6)
        traffic.setdefault(wl, {})[op] = int(rd + wr)
        out.append(f"### {wl} {op}: `{k}`\n\n")
        out.append("| metric | value |\n|---|---|\n")
        for key, (v, u) in d.items():
            out.append(f"| {key} | {v} {u} |\n")
        out.append(f"| dram read+write per launch | {(rd + wr) / 1e9:.2f} GB |\n\n")
json.dump(traffic, open(os.path.join(dst, "ncu_traffic.json"), "w"), indent=1)
open(os.path.join(dst, f"{R}_summary.md"), "w").write("".join(out))
print("".join(out))
