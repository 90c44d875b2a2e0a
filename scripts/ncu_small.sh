export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/ncu_small; mkdir -p $O
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tma_probe bench_probe/tma_gather_probe.cu -lcuda > $O/tma_build.log 2>&1
timeout 300 /tmp/tma_probe > $O/tma_probe.txt 2>&1; cat $O/tma_probe.txt
for w in "cora gcn" "pubmed gat"; do
  set -- $w
  TLP_BOTH=edge ncu --set full --import-source on --clock-control none -k regex:k_agg -s 3 -c 1 -o $O/$1 -f python scripts/one_call.py $1 $2 4 > $O/$1.log 2>&1
  ncu -i $O/$1.ncu-rep --page raw --csv > $O/$1_raw.csv 2>/dev/null
  ncu -i $O/$1.ncu-rep --page source --csv --print-source sass > $O/$1_src.csv 2>/dev/null
  rm -f $O/$1.ncu-rep
done
ls -la $O
