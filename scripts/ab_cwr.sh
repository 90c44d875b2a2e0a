# GPU box: streamed weights by cp.async into a shared-memory ring (default) vs register staging (libtlp_cwr0); then bitwise / GAT tests
bash scripts/ab_variants.sh reddit 10 base libtlp_cwr0
export TLP_SYNTH_CACHE=/tmp/tlp_synth
timeout 1500 python -m pytest tests -m gpu -x -q -k "bitwise or gat or weighted or fuzz or backward" > gpurun_out/cwr_tests.log 2>&1; tail -3 gpurun_out/cwr_tests.log
