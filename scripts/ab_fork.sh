# GPU box: GAT pre-pass on a forked stream overlapping the repack (default) vs in order (TLP_GAT_FORK=0); then the GAT / layout tests
bash scripts/ab_env.sh reddit 10 - TLP_GAT_FORK=0
export TLP_SYNTH_CACHE=/tmp/tlp_synth
timeout 1500 python -m pytest tests -m gpu -x -q -k "gat or layout or launch_counter or visit" > gpurun_out/fork_tests.log 2>&1; tail -3 gpurun_out/fork_tests.log
