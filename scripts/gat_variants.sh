export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/gatv; mkdir -p $O
for i in 1 2; do
python scripts/traffic_probe.py gat 604 10 >> $O/times.txt 2>&1
TLP_LIB_PATH=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200/libtlp_shc.so python scripts/traffic_probe.py gat 604 10 >> $O/times_shc.txt 2>&1
done
python bench.py --workload reddit_gat_bwd --no-cpu-baseline --no-e2e > $O/gatbwd.json 2>&1
TLP_LIB_PATH=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200/libtlp_shc.so python bench.py --workload reddit_gat_bwd --no-cpu-baseline --no-e2e > $O/gatbwd_shc.json 2>&1
cat $O/times.txt $O/times_shc.txt; tail -c 300 $O/gatbwd.json; tail -c 300 $O/gatbwd_shc.json
