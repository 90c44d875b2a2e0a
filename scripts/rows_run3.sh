export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/rows3; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "short_row or deterministic or launch_counter or epilogue or config_cora or config_pubmed or edge_case or feature_widths or weighted or figure1 or partition or hub or layouts" > $O/tests.log 2>&1; tail -3 $O/tests.log
cd scripts; python small_probe2.py > ../$O/probe.txt 2>&1; cd ..
grep -h "auto dynamic wpc 0 step 0\|floor" $O/probe*.txt
for w in rmat24 products; do
  python bench.py --workload $w --no-cpu-baseline --no-e2e > $O/bench_$w.json 2> $O/bench_$w.err
  TLP_ROWS=1 python bench.py --workload $w --no-cpu-baseline --no-e2e > $O/bench_${w}_rows.json 2> $O/bench_${w}_rows.err
  TLP_ROWS=1 TLP_HOT=0 python bench.py --workload $w --no-cpu-baseline --no-e2e > $O/bench_${w}_rows_nohot.json 2> $O/bench_${w}_rows_nohot.err
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/rows3/bench_*.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1])
        print(f.split('/')[-1], d["ms_per_step"], {k:v["ms_mean"] for k,v in d["ops"].items()})
    except Exception as e:
        print(f, "ERR", e)
PY
