# GPU box: k_gat_alpha scores in shared memory (default) vs in alpha[] (libtlp_as0): Reddit step A/B, kernel times, GAT tests
bash scripts/ab_variants.sh reddit 10 base libtlp_as0
export TLP_SYNTH_CACHE=/tmp/tlp_synth
L=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200
ncu --metrics gpu__time_duration.sum,lts__t_sectors.sum --clock-control none -k regex:k_gat_alpha -s 2 -c 1 --csv --log-file gpurun_out/as_base.csv python scripts/traffic_probe.py gat 604 1 > /dev/null 2>&1
TLP_LIB_PATH=$L/libtlp_as0.so ncu --metrics gpu__time_duration.sum,lts__t_sectors.sum --clock-control none -k regex:k_gat_alpha -s 2 -c 1 --csv --log-file gpurun_out/as_as0.csv python scripts/traffic_probe.py gat 604 1 > /dev/null 2>&1
for f in gpurun_out/as_*.csv; do echo "== $f"; grep -E '"(gpu__time|lts__)' $f | awk -F'","' '{print $(NF-2), $(NF-1), $NF}'; done
timeout 1200 python -m pytest tests -m gpu -x -q -k "gat" > gpurun_out/as_tests.log 2>&1; tail -3 gpurun_out/as_tests.log
