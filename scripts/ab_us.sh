# GPU box: A/B of the unit loop state in shared memory (libtlp_us) on the Reddit step + ncu spill traffic
bash scripts/ab_variants.sh reddit 10 base libtlp_us
export TLP_SYNTH_CACHE=/tmp/tlp_synth
L=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200
M=gpu__time_duration.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_write.sum,sass__inst_executed_register_spilling
for op in gin gat; do
  ncu --metrics $M --clock-control none -k regex:k_agg -s 3 -c 1 --csv python scripts/traffic_probe.py $op 604 1 > gpurun_out/us_base_$op.csv 2>&1
  TLP_LIB_PATH=$L/libtlp_us.so ncu --metrics $M --clock-control none -k regex:k_agg -s 3 -c 1 --csv python scripts/traffic_probe.py $op 604 1 > gpurun_out/us_us_$op.csv 2>&1
done
for f in gpurun_out/us_*.csv; do echo "== $f"; grep -E '"(gpu__time|dram__bytes|lts__|sass__)' $f | awk -F'","' '{print $(NF-2), $(NF-1), $NF}'; done
