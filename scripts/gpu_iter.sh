# One GPU iteration (GPU box): tests, Reddit op timings, ncu source capture of
# one kernel.  usage: bash scripts/gpu_iter.sh <tag> [pytest -k expr] [ncu op]
T=${1:-iter}; K=${2:-}; NOP=${3:-gin}
export TLP_SYNTH_CACHE=/tmp/tlp_synth
O=gpurun_out/$T; mkdir -p $O
if [ "$K" != "none" ]; then
  if [ -n "$K" ]; then timeout 1800 python -m pytest tests -m gpu -x -q -k "$K" > $O/gpu_tests.log 2>&1
  else timeout 1800 python -m pytest tests -m gpu -x -q > $O/gpu_tests.log 2>&1; fi
  tail -3 $O/gpu_tests.log
fi
for op in gin gcn_both gat; do python scripts/traffic_probe.py $op 604 10 >> $O/times.txt 2>&1; done
cat $O/times.txt
if [ "$NOP" != "none" ]; then
  ncu --set full --import-source on --clock-control none -k regex:k_agg -s 3 -c 1 -o $O/prof -f \
    python scripts/traffic_probe.py $NOP 604 1 > $O/ncu.log 2>&1
  ncu -i $O/prof.ncu-rep --page raw --csv > $O/raw.csv 2>/dev/null
  ncu -i $O/prof.ncu-rep --page source --csv --print-source sass > $O/source_sass.csv 2>/dev/null
  ls -la $O
fi
