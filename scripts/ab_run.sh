# A/B of two library builds on the Reddit ops: times (2 rounds) + ncu DRAM bytes of each k_agg
export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/ab; mkdir -p $O
L=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200
B=${1:-libtlp_smrp}
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_op_write.sum,lts__throughput.avg.pct_of_peak_sustained_elapsed
for i in 1 2; do for op in gin gcn_both gat; do
  python scripts/traffic_probe.py $op 604 10 >> $O/times_base.txt 2>&1
  TLP_LIB_PATH=$L/$B.so python scripts/traffic_probe.py $op 604 10 >> $O/times_$B.txt 2>&1
done; done
for op in gin gcn_both gat; do
  ncu --metrics $M --clock-control none -k regex:k_agg -s 3 -c 1 --csv python scripts/traffic_probe.py $op 604 1 > $O/ncu_base_$op.csv 2>&1
  TLP_LIB_PATH=$L/$B.so ncu --metrics $M --clock-control none -k regex:k_agg -s 3 -c 1 --csv python scripts/traffic_probe.py $op 604 1 > $O/ncu_${B}_$op.csv 2>&1
done
cat $O/times_base.txt $O/times_$B.txt | awk '{print $1, $NF, $0}' | cut -c1-60
for f in $O/ncu_*.csv; do echo "== $f"; grep -E '"(gpu__time|dram__bytes|lts__)' $f | awk -F'","' '{print $(NF-2), $(NF-1), $NF}'; done
