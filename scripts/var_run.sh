export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/var1; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "gather_paths or hub or rmat or products or short_row or lane_groups or gat_backward or alpha" > $O/tests.log 2>&1; tail -3 $O/tests.log
TLP_LIB_PATH=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200/libtlp_shc.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "lane_groups or gat_backward or alpha or panel or layouts" > $O/tests_shc.log 2>&1; tail -3 $O/tests_shc.log
for i in 1 2; do
python scripts/traffic_probe.py gat 604 10 >> $O/times.txt 2>&1
TLP_LIB_PATH=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200/libtlp_shc.so python scripts/traffic_probe.py gat 604 10 >> $O/times_shc.txt 2>&1
done
for w in rmat24 products products_gat4; do python bench.py --workload $w --no-cpu-baseline --no-e2e > $O/bench_$w.json 2> $O/bench_$w.err; done
python bench.py --workload reddit_gat_bwd --no-cpu-baseline --no-e2e > $O/gatbwd.json 2>&1
TLP_LIB_PATH=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200/libtlp_shc.so python bench.py --workload reddit_gat_bwd --no-cpu-baseline --no-e2e > $O/gatbwd_shc.json 2>&1
cat $O/times.txt $O/times_shc.txt
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/var1/*.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); print(f.split('/')[-1], d["ms_per_step"], {k:v["ms_mean"] for k,v in d["ops"].items()})
    except Exception as e: print(f, "ERR", e)
PY
