# GPU box: full -m gpu suite, smoke, small-config bench lines.  usage: bash scripts/gpu_suite.sh <tag>
O=gpurun_out/${1:-suite}; mkdir -p $O
export TLP_SYNTH_CACHE=/tmp/tlp_synth
timeout 3000 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; tail -4 $O/gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
for w in cora pubmed; do
  timeout 900 python bench.py --workload $w --no-cpu-baseline --steps 4000 --warmup 100 > $O/bench_$w.json 2> $O/bench_$w.err
  python -c "import json; d=json.loads(open('$O/bench_$w.json').read().strip().splitlines()[-1]); print('$w', d['ms_per_step'], {k: v['ms_mean'] for k, v in d['ops'].items()}, d['roofline']['frac'], d['clocks'])"
done
