# GPU box: short-row kernel probe + its parity tests (+ the full -m gpu suite with "full").
O=gpurun_out/${1:-rows}; mkdir -p $O
export TLP_SYNTH_CACHE=/tmp/tlp_synth
(cd scripts && timeout 600 python rows_probe.py > ../$O/rows_probe.txt 2>&1); tail -40 $O/rows_probe.txt
timeout 900 python -m pytest tests -m gpu -x -q -k "short_row or launch_counter or visit_counter" > $O/rows_tests.log 2>&1; tail -3 $O/rows_tests.log
if [ "$2" = "full" ]; then timeout 3000 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; tail -5 $O/gpu_tests.log; fi
