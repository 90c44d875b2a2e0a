export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/depth; mkdir -p $O
L=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200
for v in libtlp libtlp_d12 libtlp_d20 libtlp_d12b4; do
  for w in products rmat24 products_gat4; do
    TLP_LIB_PATH=$L/$v.so timeout 600 python bench.py --workload $w --no-cpu-baseline --no-e2e > $O/${v}_$w.json 2> $O/${v}_$w.err
  done
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/depth/*.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); print(f.split('/')[-1], d["ms_per_step"], d["clocks"]["sm_mhz"])
    except Exception as e: print(f, "ERR", e)
PY
