export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/small3; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "short_row or deterministic or launch_counter or epilogue or config_cora or config_pubmed or edge_case or feature_widths or weighted or figure1" > $O/tests.log 2>&1; tail -3 $O/tests.log
cd scripts
python small_probe2.py > ../$O/probe_default.txt 2>&1
TLP_LIB_PATH=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200/libtlp_rows48.so python small_probe2.py > ../$O/probe_rows48.txt 2>&1
TLP_ROWS=0 python small_probe2.py > ../$O/probe_norows.txt 2>&1
cd ..; grep -h "auto dynamic wpc 0 step 0\|floor" $O/probe_*.txt
