# GPU box: default (coefficients by shuffle) vs the shared-memory row (libtlp_smc1); then the full -m gpu suite on the default
bash scripts/ab_variants.sh reddit 10 base libtlp_smc1
export TLP_SYNTH_CACHE=/tmp/tlp_synth
timeout 3000 python -m pytest tests -m gpu -q > gpurun_out/shc2_tests.log 2>&1; tail -3 gpurun_out/shc2_tests.log
