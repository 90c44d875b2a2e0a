"""Summarise a round's ncu evidence (raw CSV pages brought back from the GPU box
by scripts/evidence_r02.sh) and bench lines into profiles/ (tracked):
profiles/<R>_summary.md, profiles/<R>_bench*.json, profiles/<R>_launches.csv,
profiles/<R>_ncu_<name>.csv and profiles/ncu_traffic.json (DRAM bytes per
launch that bench.py reports as roofline.traffic).

usage: python scripts/summarize_profiles.py r02"""
import csv
import glob
import json
import os
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
R = sys.argv[1] if len(sys.argv) > 1 else "r02"
SRC = os.path.join(ROOT, "gpurun_out", R)
DST = os.path.join(ROOT, "profiles")

METRICS = [
    ("time", "gpu__time_duration.sum"),
    ("dram_rd", "dram__bytes_read.sum"),
    ("dram_wr", "dram__bytes_write.sum"),
    ("dram_%", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"),
    ("l2_hit_%", "lts__t_sector_hit_rate.pct"),
    ("l2_sectors", "lts__t_sectors.sum"),
    ("l2_throughput_%", "lts__throughput.avg.pct_of_peak_sustained_elapsed"),
    ("l1_hit_%", "l1tex__t_sector_hit_rate.pct"),
    ("occupancy_%", "sm__warps_active.avg.pct_of_peak_sustained_active"),
    ("issue_active_%", "smsp__issue_active.avg.pct_of_peak_sustained_active"),
    ("inst", "smsp__inst_executed.sum"),
    ("regs", "launch__registers_per_thread"),
    ("grid", "launch__grid_size"),
    ("block", "launch__block_size"),
    ("local_ld_sectors", "lts__t_sectors_srcunit_tex_aperture_device_op_read.sum"),
]
# (capture name -> (workload key in ncu_traffic.json, op))
TRAFFIC_KEYS = {
    "reddit_gcn": ("reddit", "gcn"), "reddit_gin": ("reddit", "gin"), "reddit_gat": ("reddit", "gat"),
    "reddit_gat_alpha": ("reddit", "gat_alpha"), "reddit_repack": ("reddit", "repack"),
    "reddit_gat_online": ("reddit", "gat_online"), "products_gat": ("products", "gat"), "products_gat4": ("products", "gat4"),
    "rmat24_gcn": ("rmat24", "gcn"), "cora_gcn": ("cora", "gcn"), "pubmed_gat": ("pubmed", "gat"),
}


def to_bytes(v, unit):
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)
    return float(v) * scale


def read_raw(path):
    rows = list(csv.reader(open(path)))
    if len(rows) < 3:
        return None
    h, u, d = rows[0], rows[1], rows[2]
    out = {"kernel": d[h.index("Kernel Name")] if "Kernel Name" in h else "?"}
    for key, m in METRICS:
        if m in h:
            out[key] = (d[h.index(m)].replace(",", ""), u[h.index(m)])
    stalls = []
    for i, name in enumerate(h):
        if name.startswith("smsp__average_warps_issue_stalled_") and name.endswith("_per_issue_active.ratio"):
            try:
                stalls.append((float(d[i]), name[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
            except ValueError:
                pass
    out["top_stalls"] = sorted(stalls, reverse=True)[:4]
    return out


def main():
    os.makedirs(DST, exist_ok=True)
    md = [f"# Round {R} profile summary\n\n"]
    # bench lines
    bj = os.path.join(SRC, "bench.json")
    if os.path.exists(bj):
        b = json.loads(open(bj).read().strip().splitlines()[-1])
        json.dump(b, open(os.path.join(DST, f"{R}_bench.json"), "w"), indent=1)
        md.append("## bench.py (default: Reddit-shaped GCN + GIN + GAT step)\n\n")
        md.append(f"value {b['value']} GB/s gather-model, {b['ms_per_step']} ms/step, clocks {b['clocks']}\n\n")
        for op, d in b["ops"].items():
            md.append(f"* {op}: {d['ms_mean']} ms mean ({d['gather_GBs']} GB/s gather-model)\n")
        md.append(f"\nroofline: {json.dumps(b['roofline'])}\n\n")
        if b.get("cpu_baseline"):
            md.append(f"cpu_baseline: {json.dumps(b['cpu_baseline'])}\n\n")
    extra = sorted(glob.glob(os.path.join(SRC, "bench_*.json")))
    if extra:
        md.append("## other workloads (bench.py --workload W)\n\n")
        md.append("| workload | ms/step | per op ms (mean) | GB/s gather-model | roofline bound / frac | e2e GB/s | sm MHz (samples) |\n")
        md.append("|---|---|---|---|---|---|---|\n")
        for f in extra:
            try:
                b = json.loads(open(f).read().strip().splitlines()[-1])
            except Exception:
                continue
            wl = os.path.basename(f)[6:-5]
            json.dump(b, open(os.path.join(DST, f"{R}_bench_{wl}.json"), "w"), indent=1)
            ops = ", ".join(f"{k} {v['ms_mean']}" for k, v in b.get("ops", {}).items())
            e2e = (b.get("e2e") or {}).get("value")
            rf = b.get("roofline", {})
            md.append(f"| {wl} | {b['ms_per_step']} | {ops} | {b['value']} | {rf.get('bound')} {rf.get('frac')} "
                      f"| {e2e} | {b['clocks']['sm_mhz']} ({b['clocks'].get('samples')}) |\n")
            if b.get("paper_context"):
                md.append(f"| ↳ paper V100 (F=32) | | {b['paper_context']['v100_ms']} | B200/V100 "
                          f"{b['paper_context']['b200_over_v100']} | | | |\n")
        md.append("\n")
    # launch list
    lc = os.path.join(SRC, "launches.csv")
    if os.path.exists(lc):
        rows = list(csv.reader(open(lc)))
        start = next((i for i, r in enumerate(rows) if r and r[0] == "ID"), None)
        if start is not None:
            hdr = rows[start]
            ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
            tot, cnt = defaultdict(float), defaultdict(int)
            for r in rows[start + 1:]:
                if len(r) > vi:
                    tot[r[ki]] += float(r[vi].replace(",", ""))
                    cnt[r[ki]] += 1
            ours = {k: v for k, v in tot.items() if any(x in k for x in ("k_agg", "k_repack", "k_gat_alpha", "k_rows"))}
            T = sum(ours.values())
            md.append("## ncu launch list of the bench step (gpu__time_duration.sum; cold-cache, serialised)\n\n")
            for k, v in sorted(ours.items(), key=lambda x: -x[1]):
                md.append(f"* `{k}`: {v / 1e6 / cnt[k]:.3f} ms per launch, {cnt[k]} launches, "
                          f"{100 * v / T:.1f} % of the step's kernel time\n")
            md.append("\n")
            open(os.path.join(DST, f"{R}_launches.csv"), "w").write(open(lc).read())
    # ncu --set full captures
    traffic = {}
    p = os.path.join(DST, "ncu_traffic.json")
    if os.path.exists(p):
        traffic = json.load(open(p))
    md.append("## ncu --set full (one launch each, --clock-control none, cold caches)\n\n")
    for raw in sorted(glob.glob(os.path.join(SRC, "*_raw.csv"))):
        name = os.path.basename(raw)[:-8]
        d = read_raw(raw)
        if d is None:
            continue
        open(os.path.join(DST, f"{R}_ncu_{name}.csv"), "w").write(open(raw).read())
        rd = to_bytes(*d["dram_rd"]) if "dram_rd" in d else 0.0
        wr = to_bytes(*d["dram_wr"]) if "dram_wr" in d else 0.0
        if name in TRAFFIC_KEYS:
            wl, op = TRAFFIC_KEYS[name]
            traffic.setdefault(wl, {})[op] = int(rd + wr)
        md.append(f"### {name}: `{d['kernel'][:110]}`\n\n| metric | value |\n|---|---|\n")
        for key, _ in METRICS:
            if key in d:
                md.append(f"| {key} | {d[key][0]} {d[key][1]} |\n")
        md.append(f"| dram read + write per launch | {(rd + wr) / 1e9:.3f} GB |\n")
        md.append("| top stalls (per issued instruction) | " +
                  ", ".join(f"{n} {v:.2f}" for v, n in d["top_stalls"]) + " |\n\n")
    json.dump(traffic, open(p, "w"), indent=1)
    open(os.path.join(DST, f"{R}_summary.md"), "w").write("".join(md))
    print("".join(md))


if __name__ == "__main__":
    main()
