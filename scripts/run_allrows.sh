export TLP_SYNTH_CACHE=/tmp/tlp_synth
mkdir -p gpurun_out/allrows
nproc > gpurun_out/allrows/nproc.txt
timeout 2400 python -m pytest tests/test_config_allrows.py tests/test_dist_torchrun.py tests/test_gpu_parity.py -k "allrows or torchrun or layouts or reddit or products" -m gpu -q --durations=20 > gpurun_out/allrows/tests.log 2>&1
tail -40 gpurun_out/allrows/tests.log
