# GPU box: final bench lines of the default step and the multi-head workload, plus the mh parity tests
O=gpurun_out/final2; mkdir -p $O
export TLP_SYNTH_CACHE=/tmp/tlp_synth
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
timeout 900 python bench.py --workload products_gat4 --no-cpu-baseline --steps 60 > $O/bench_products_gat4.json 2> $O/bench_products_gat4.err
timeout 900 python bench.py --workload products --no-cpu-baseline --steps 60 > $O/bench_products.json 2> $O/bench_products.err
for f in $O/bench*.json; do python -c "import json; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', d['ms_per_step'], {k: v['ms_mean'] for k, v in d['ops'].items()}, d['roofline']['frac'], d['clocks'])"; done
