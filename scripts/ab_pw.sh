# GPU box: multi-head async pair weights as float2 ahead of the wait (default) vs per-edge reads (libtlp_pw0); then the multi-head tests
bash scripts/ab_variants.sh products_gat4 40 base libtlp_pw0
export TLP_SYNTH_CACHE=/tmp/tlp_synth
timeout 1200 python -m pytest tests -m gpu -x -q -k "mh or multi_head or gat4 or fuzz" > gpurun_out/pw_tests.log 2>&1; tail -3 gpurun_out/pw_tests.log
