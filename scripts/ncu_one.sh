# GPU box: ncu --set full (with source counters) of one kernel of one config call.
# usage: bash scripts/ncu_one.sh <tag> <name> <kernel regex> <workload> <op> [env...]
O=gpurun_out/$1; mkdir -p $O; n=$2; k=$3; w=$4; op=$5; shift 5
export TLP_SYNTH_CACHE=/tmp/tlp_synth
env "$@" python scripts/one_call.py $w $op 1 > /dev/null 2>&1
env "$@" ncu --set full --import-source on --clock-control none -k regex:$k -s 3 -c 1 -o $O/$n -f python scripts/one_call.py $w $op 4 > $O/$n.log 2>&1
ncu -i $O/$n.ncu-rep --page raw --csv > $O/${n}_raw.csv 2>/dev/null
ncu -i $O/$n.ncu-rep --page source --csv --print-source sass > $O/${n}_sass.csv 2>/dev/null
ncu -i $O/$n.ncu-rep --page details --csv > $O/${n}_details.csv 2>/dev/null
rm -f $O/$n.ncu-rep
