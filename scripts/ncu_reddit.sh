# GPU box: ncu --set full with source counters of one Reddit panel kernel.
# usage: bash scripts/ncu_reddit.sh <tag> <op: gin|gcn_both|gat>
O=gpurun_out/$1; mkdir -p $O; op=$2
export TLP_SYNTH_CACHE=/tmp/tlp_synth
python scripts/traffic_probe.py $op 604 1 > /dev/null 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_agg -s 3 -c 1 -o $O/reddit_$op -f python scripts/traffic_probe.py $op 604 1 > $O/reddit_$op.log 2>&1
ncu -i $O/reddit_$op.ncu-rep --page source --csv --print-source sass > $O/reddit_${op}_sass.csv 2>/dev/null
ncu -i $O/reddit_$op.ncu-rep --page details --csv > $O/reddit_${op}_details.csv 2>/dev/null
rm -f $O/reddit_$op.ncu-rep
