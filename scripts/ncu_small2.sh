export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/ncu_small2; mkdir -p $O
for w in "cora gcn" "pubmed gat"; do
  set -- $w
  ncu --set full --import-source on --clock-control none -k regex:k_rows -s 3 -c 1 -o $O/$1 -f python scripts/one_call.py $1 $2 4 > $O/$1.log 2>&1
  ncu -i $O/$1.ncu-rep --page raw --csv > $O/$1_raw.csv 2>/dev/null
  ncu -i $O/$1.ncu-rep --page source --csv --print-source sass > $O/$1_src.csv 2>/dev/null
  rm -f $O/$1.ncu-rep
done
ls -la $O
