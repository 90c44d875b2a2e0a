# GPU box: ncu --set full (with source counters) of the short-row kernel on Cora GCN and Pubmed GAT.
O=gpurun_out/${1:-ncu_small}; mkdir -p $O
export TLP_SYNTH_CACHE=/tmp/tlp_synth
for w in "cora gcn" "pubmed gat"; do
  set -- $w
  python scripts/one_call.py $1 $2 4 > /dev/null 2>&1
  ncu --set full --import-source on --clock-control none -k regex:k_rows -s 3 -c 1 -o $O/${1}_$2 -f python scripts/one_call.py $1 $2 4 > $O/${1}_$2.log 2>&1
  ncu -i $O/${1}_$2.ncu-rep --page raw --csv > $O/${1}_${2}_raw.csv 2>/dev/null
  ncu -i $O/${1}_$2.ncu-rep --page source --csv --print-source sass > $O/${1}_${2}_sass.csv 2>/dev/null
  ncu -i $O/${1}_$2.ncu-rep --page details --csv > $O/${1}_${2}_details.csv 2>/dev/null
  rm -f $O/${1}_$2.ncu-rep
done
ls -la $O
