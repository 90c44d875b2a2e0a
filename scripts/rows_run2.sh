export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/rows2; mkdir -p $O
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tma_probe bench_probe/tma_gather_probe.cu -lcuda > $O/tma_build.log 2>&1
timeout 300 /tmp/tma_probe > $O/tma_probe.txt 2>&1; cat $O/tma_probe.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "short_row or deterministic or launch_counter or epilogue or config_cora or config_pubmed or edge_case or feature_widths or weighted or figure1 or partition or hub" > $O/tests.log 2>&1; tail -3 $O/tests.log
cd scripts; python small_probe2.py > ../$O/probe.txt 2>&1; TLP_ROWS_MAJOR=0 python small_probe2.py > ../$O/probe_major0.txt 2>&1; cd ..
grep -h "auto dynamic wpc 0 step 0\|floor" $O/probe*.txt
for v in "alpha" "online" "online64"; do
  case $v in alpha) E="";; online) E="TLP_GAT=online";; online64) E="TLP_GAT=online TLP_PANEL=64";; esac
  env $E python scripts/traffic_probe.py gat 604 10 >> $O/gat.txt 2>&1
done
cat $O/gat.txt
