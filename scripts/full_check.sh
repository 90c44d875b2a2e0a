# GPU box: full -m gpu suite, smoke, bench lines (default + config workloads).
T=${1:-chk}; O=gpurun_out/$T; mkdir -p $O
export TLP_SYNTH_CACHE=/tmp/tlp_synth
timeout 2400 python -m pytest tests -m gpu -x -q > $O/gpu_tests.log 2>&1; tail -3 $O/gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
for w in products rmat24 products_gat4; do timeout 900 python bench.py --workload $w --no-cpu-baseline > $O/bench_$w.json 2> $O/bench_$w.err; done
for w in cora pubmed; do timeout 900 python bench.py --workload $w --no-cpu-baseline --steps 4000 --warmup 100 > $O/bench_$w.json 2> $O/bench_$w.err; done
python - <<PY
import json, glob
for f in sorted(glob.glob("$O/bench*.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); print(f.split('/')[-1], d["value"], d["ms_per_step"], {k:v["ms_mean"] for k,v in d["ops"].items()}, d["roofline"]["bound"], d["roofline"]["frac"], d["clocks"]["sm_mhz"], d.get("create_ms"))
    except Exception as e: print(f, "ERR", e)
PY
