# GPU box: multi-head head-index multiply-high (default) vs integer division (libtlp_div); then the multi-head tests
bash scripts/ab_variants.sh products_gat4 40 base libtlp_div
export TLP_SYNTH_CACHE=/tmp/tlp_synth
timeout 1200 python -m pytest tests -m gpu -x -q -k "mh or multi_head or gat4 or fuzz" > gpurun_out/div_tests.log 2>&1; tail -3 gpurun_out/div_tests.log
