# A/B of environment knobs on one bench workload (GPU box), interleaved rounds.
# usage: bash scripts/ab_env.sh <workload> <steps> "<env1>" "<env2>" ...   ("-" = defaults)
W=$1; K=$2; shift 2
export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/abenv_$W; mkdir -p $O
for i in 1 2 3; do
  n=0
  for v in "$@"; do
    n=$((n+1))
    if [ "$v" = "-" ]; then ev=""; else ev="$v"; fi
    env $ev timeout 600 python bench.py --workload $W --no-cpu-baseline --no-e2e --steps $K > $O/v$n.$i.json 2>$O/v$n.err
    python -c "import json;b=json.loads(open('$O/v$n.$i.json').read().splitlines()[-1]);print('$v', $i, b['ms_per_step'], {k: v['ms_mean'] for k, v in b['ops'].items()}, b['clocks']['sm_mhz'])"
  done
done
