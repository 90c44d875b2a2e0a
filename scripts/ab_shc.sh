# GPU box: lane-group coefficients by shuffle (libtlp_shc, TLP_SMEMC=2) vs the shared-memory row (base): GAT backward A/B + tests on the variant
bash scripts/ab_variants.sh reddit_gat_bwd 6 base libtlp_shc
bash scripts/ab_variants.sh reddit 10 base libtlp_shc
export TLP_SYNTH_CACHE=/tmp/tlp_synth
TLP_LIB_PATH=$GRAFT_REPO_ROOT/paper_conf_hpdc_fujh22_b200/libtlp_shc.so timeout 1500 python -m pytest tests -m gpu -x -q -k "bitwise or gat or weighted or fuzz or backward or panel" > gpurun_out/shc_tests.log 2>&1; tail -3 gpurun_out/shc_tests.log
