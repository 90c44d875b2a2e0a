# GPU box: full -m gpu suite, smoke, default bench line.  usage: bash scripts/gpu_check.sh <tag>
T=${1:-check}; O=gpurun_out/$T; mkdir -p $O
export TLP_SYNTH_CACHE=/tmp/tlp_synth
timeout 2400 python -m pytest tests -m gpu -x -q > $O/gpu_tests.log 2>&1; tail -3 $O/gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -2 $O/smoke.log
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err; tail -c 1500 $O/bench.json
