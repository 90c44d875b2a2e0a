export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/small4; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "short_row or deterministic or launch_counter or epilogue or config_cora or config_pubmed or edge_case or feature_widths or weighted or figure1 or partition" > $O/tests.log 2>&1; tail -3 $O/tests.log
python scripts/host_probe.py > $O/host.txt 2>&1; cat $O/host.txt
cd scripts; python small_probe2.py > ../$O/probe.txt 2>&1; TLP_GAT=alpha python small_probe2.py > ../$O/probe_alpha.txt 2>&1; cd ..
grep -h "auto dynamic wpc 0 step 0\|floor" $O/probe*.txt
for w in cora pubmed; do python bench.py --workload $w --no-cpu-baseline > $O/bench_$w.json 2> $O/bench_$w.err; done
python - <<'PY'
import json
for w in ("cora","pubmed"):
    d=json.loads(open(f"gpurun_out/small4/bench_{w}.json").read().strip().splitlines()[-1])
    print(w, d["ms_per_step"], {k:v["ms_mean"] for k,v in d["ops"].items()}, d["roofline"]["frac"], d["clocks"])
PY
