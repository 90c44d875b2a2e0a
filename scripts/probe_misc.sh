# GPU box: (1) Reddit step, gathers with / without L1 allocation (libtlp_l1na);
# (2) their L2 write sectors, local-memory (spill) traffic and DRAM bytes;
# (3) products 4-head GAT, register vs cp.async gather path.
O=gpurun_out/misc; mkdir -p $O
export TLP_SYNTH_CACHE=/tmp/tlp_synth
L=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200
bash scripts/ab_variants.sh reddit 10 base libtlp_l1na
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_write.sum,l1tex__t_sectors_pipe_lsu_mem_local_op_st_lookup_miss.sum,lts__throughput.avg.pct_of_peak_sustained_elapsed
for op in gin gat gcn_both; do
  ncu --metrics $M --clock-control none -k regex:k_agg -s 3 -c 1 --csv python scripts/traffic_probe.py $op 604 1 > $O/ncu_base_$op.csv 2>&1
  TLP_LIB_PATH=$L/libtlp_l1na.so ncu --metrics $M --clock-control none -k regex:k_agg -s 3 -c 1 --csv python scripts/traffic_probe.py $op 604 1 > $O/ncu_l1na_$op.csv 2>&1
done
for f in $O/ncu_*.csv; do echo "== $f"; grep -E '"(gpu__time|dram__bytes|lts__|l1tex__)' $f | awk -F'","' '{print $(NF-2), $(NF-1), $NF}'; done
for i in 1 2; do
  timeout 600 python bench.py --workload products_gat4 --no-cpu-baseline --no-e2e --steps 40 > $O/gat4_async.$i.json 2>/dev/null
  TLP_GATHER=reg timeout 600 python bench.py --workload products_gat4 --no-cpu-baseline --no-e2e --steps 40 > $O/gat4_reg.$i.json 2>/dev/null
done
for f in $O/gat4_*.json; do python -c "import json;b=json.loads(open('$f').read().splitlines()[-1]);print('$f', b['ms_per_step'], b['clocks']['sm_mhz'])"; done
