mkdir -p gpurun_out
for m in ${1:-"128 64"}; do
  TLP_PANEL=$m python bench.py --workload reddit --steps 8 --no-e2e --no-cpu-baseline > gpurun_out/bp_$m.json 2>gpurun_out/bp_$m.err
  python -c "import json;d=json.load(open('gpurun_out/bp_$m.json'));print('panel $m', d['value'],{k:v['ms_mean'] for k,v in d['ops'].items()}, d['clocks']['sm_mhz'])" 2>&1 | tail -1
done
