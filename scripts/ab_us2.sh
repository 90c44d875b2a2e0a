# GPU box: unit loop state in shared memory for the coefficient-free sums (default) vs off (libtlp_us0); then the bitwise / parity tests
bash scripts/ab_variants.sh reddit 10 base libtlp_us0
bash scripts/ab_variants.sh reddit_sage 6 base libtlp_us0
export TLP_SYNTH_CACHE=/tmp/tlp_synth
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/us2_tests.log 2>&1; tail -3 gpurun_out/us2_tests.log
