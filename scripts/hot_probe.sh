# Hot-source L2 policy sweep.
# usage: bash scripts/hot_probe.sh "<workloads>" "<fractions>"
mkdir -p gpurun_out/hot
W=${1:-"products"}
FR=${2:-"none 0.3 0.5 0.7"}
for w in $W; do
  for f in $FR; do
    for c in 0 1; do
      if [ "$f" = "none" ]; then [ $c = 1 ] && continue; unset TLP_HOT; else export TLP_HOT=$f; fi
      export TLP_HOT_COLD=$c
      python bench.py --workload $w --steps 8 --no-e2e --no-cpu-baseline > gpurun_out/hot/${w}_${f}_$c.json 2>gpurun_out/hot/${w}_${f}_$c.err
      python -c "import json;d=json.load(open('gpurun_out/hot/${w}_${f}_$c.json'));print('$w hot=$f cold_first=$c', d['value'],{k:v['ms_mean'] for k,v in d['ops'].items()}, d['clocks']['sm_mhz'])" 2>&1 | tail -1
    done
  done
done
unset TLP_HOT TLP_HOT_COLD
