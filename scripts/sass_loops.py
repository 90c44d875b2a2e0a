"""Innermost-loop sizes of a kernel's SASS (offline, no GPU): compiles one
csrc translation unit for sm_100a, disassembles it and prints, for every
backward branch whose body contains the given marker instruction (default
LDGDEPBAR: the cp.async pipeline loops), the body's instruction count.
usage: python scripts/sass_loops.py <tlp_k_x.cu> <kernel-name regex> [marker] [-D...]"""
import os, re, subprocess, sys, tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_hpdc_fujh22_b200", "csrc")
src, pat = sys.argv[1], sys.argv[2]
marker = sys.argv[3] if len(sys.argv) > 3 and not sys.argv[3].startswith("-D") else "LDGDEPBAR"
defs = [a for a in sys.argv[3:] if a.startswith("-D")]
cubin = os.path.join(tempfile.mkdtemp(), "k.cubin")
subprocess.run(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-std=c++17", "-cubin",
                "-I" + os.path.join(ROOT, "include"), *defs, "-o", cubin, os.path.join(CSRC, src)], check=True)
sass = subprocess.run(["cuobjdump", "-sass", cubin], capture_output=True, text=True).stdout
funcs = re.split(r"\n\s*Function : ", sass)
for f in funcs[1:]:
    name = f.split("\n", 1)[0].strip()
    dem = subprocess.run(["c++filt", name], capture_output=True, text=True).stdout.strip()
    if not re.search(pat, dem):
        continue
    ins = []  # (addr, text)
    for line in f.split("\n"):
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s*(.*?);", line)
        if m:
            ins.append((int(m.group(1), 16), m.group(2).strip()))
    idx = {a: i for i, (a, _) in enumerate(ins)}
    print(f"== {dem}  ({len(ins)} instructions)")
    back = []  # backward branches (loops)
    for i, (a, t) in enumerate(ins):
        m = re.search(r"BRA\s+(?:`\()?.*?0x([0-9a-f]+)", t)
        if m and int(m.group(1), 16) < a and int(m.group(1), 16) in idx:
            back.append((idx[int(m.group(1), 16)], i))
    for lo, hi in back:
        if any(lo <= l2 and h2 <= hi and (l2, h2) != (lo, hi) for l2, h2 in back):
            continue  # not innermost
        tgt, a = ins[lo][0], ins[hi][0]
        if True:
            body = ins[lo:hi + 1]
            if any(marker in x for _, x in body):
                print(f"  loop {tgt:#x}-{a:#x}: {len(body)} instructions, "
                      f"{sum('LDGSTS' in x for _, x in body)} LDGSTS, {sum('SHFL' in x for _, x in body)} SHFL, "
                      f"{sum(x.startswith('FFMA') or ' FFMA' in x for _, x in body)} FFMA")
                if os.environ.get("SHOW"):
                    for _, x in body:
                        print("     ", x)
