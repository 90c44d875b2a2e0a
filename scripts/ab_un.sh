# GPU box: k_gat_alpha edges per thread per step (TLP_ALPHA_UN 8 default vs 4 / 16): kernel time by ncu, Reddit GAT
export TLP_SYNTH_CACHE=/tmp/tlp_synth
L=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200
python scripts/traffic_probe.py gat 604 1 > /dev/null 2>&1
for v in base libtlp_un4 libtlp_un16; do
  if [ "$v" = base ]; then unset TLP_LIB_PATH; else export TLP_LIB_PATH=$L/$v.so; fi
  ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_gat_alpha -s 2 -c 3 --csv --log-file gpurun_out/un_$v.csv python scripts/traffic_probe.py gat 604 2 > /dev/null 2>&1
  echo "$v $(grep gpu__time gpurun_out/un_$v.csv | awk -F'","' '{print $NF}' | tr -d '"' | tr '\n' ' ')"
done
