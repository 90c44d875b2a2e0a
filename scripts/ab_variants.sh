# A/B of in-tree library variants on one bench workload (GPU box), interleaved
# rounds so drift under the power cap hits every variant alike.
# usage: bash scripts/ab_variants.sh <workload> <steps> <variant...>   (variant: base | libtlp_X)
W=$1; K=$2; shift 2
export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/ab_$W; mkdir -p $O
L=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200
for i in 1 2 3; do
  for v in "$@"; do
    if [ "$v" = base ]; then unset TLP_LIB_PATH; else export TLP_LIB_PATH=$L/$v.so; fi
    timeout 600 python bench.py --workload $W --no-cpu-baseline --no-e2e --steps $K > $O/$v.$i.json 2>$O/$v.err
    python -c "import json;b=json.loads(open('$O/$v.$i.json').read().splitlines()[-1]);print('$v', $i, b['ms_per_step'], {k: v['ms_mean'] for k, v in b['ops'].items()}, b['clocks']['sm_mhz'])"
  done
done
unset TLP_LIB_PATH
