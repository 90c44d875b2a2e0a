# usage (GPU box): bash scripts/layout_run.sh -> gpurun_out/layout/*
export TLP_SYNTH_CACHE=/tmp/tlp_synth
mkdir -p gpurun_out/layout
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/layout/gpu_tests.log 2>&1
for op in gin gcn_both gat; do
  for lay in caller padded panel; do
    TLP_LAYOUT=$lay python scripts/traffic_probe.py $op 604 10 >> gpurun_out/layout/times.txt 2>&1
  done
  python scripts/traffic_probe.py $op 608 10 >> gpurun_out/layout/times.txt 2>&1
done
