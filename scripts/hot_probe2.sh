# register-path vs cp.async-path gathers under the hot-source policy (products GAT)
mkdir -p gpurun_out/hot2
export TLP_SYNTH_CACHE=/tmp/tlp_synth
for gp in reg async; do
  for f in none 0.5; do
    if [ "$f" = "none" ]; then unset TLP_HOT; else export TLP_HOT=$f; fi
    export TLP_HOT_COLD=1 TLP_GATHER=$gp
    python bench.py --workload products --steps 8 --no-e2e --no-cpu-baseline > gpurun_out/hot2/p_${gp}_$f.json 2>gpurun_out/hot2/p_${gp}_$f.err
    python -c "import json;d=json.load(open('gpurun_out/hot2/p_${gp}_$f.json'));print('products $gp hot=$f', d['value'],{k:v['ms_mean'] for k,v in d['ops'].items()}, d['clocks']['sm_mhz'])" 2>&1 | tail -1
  done
done
unset TLP_HOT TLP_HOT_COLD TLP_GATHER
