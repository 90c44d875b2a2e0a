# GPU box: A/B of the half-warp-major coefficient row (default) vs per-step reads (libtlp_c2off)
bash scripts/ab_variants.sh reddit 10 base libtlp_c2off
bash scripts/ab_variants.sh reddit_gat_bwd 6 base libtlp_c2off
export TLP_SYNTH_CACHE=/tmp/tlp_synth
timeout 1200 python -m pytest tests -m gpu -x -q -k "bitwise or gat_alpha or reddit_gat or backward" > gpurun_out/ab_c2_tests.log 2>&1; tail -3 gpurun_out/ab_c2_tests.log
