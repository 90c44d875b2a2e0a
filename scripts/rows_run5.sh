export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/rows5; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "short_row or gat or hub or figure1 or edge_case" > $O/tests.log 2>&1; tail -3 $O/tests.log
cd scripts
python small_probe2.py > ../$O/probe_u6.txt 2>&1
for u in 4 8; do TLP_LIB_PATH=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200/libtlp_u$u.so python small_probe2.py > ../$O/probe_u$u.txt 2>&1; done
cd ..
for f in $O/probe*.txt; do echo "== $f"; grep -h "auto dynamic wpc 0 step 0" $f; done
