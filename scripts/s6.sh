mkdir -p gpurun_out/s6
export TLP_SYNTH_CACHE=/tmp/tlp_synth
S=gpurun_out/s6/summary.txt
b() {  # <tag> <bench args...>
  t=$1; shift
  python bench.py "$@" > gpurun_out/s6/$t.json 2> gpurun_out/s6/$t.err
  python -c "import json;d=json.load(open('gpurun_out/s6/$t.json'));print('$t', d['value'], d['ms_per_step'], {k:v['ms_mean'] for k,v in d['ops'].items()}, d['clocks']['sm_mhz'])" >> $S 2>&1
}
b reddit --steps 6 --no-e2e --no-cpu-baseline
b reddit_bwd --workload reddit_bwd --steps 6 --no-e2e --no-cpu-baseline
b reddit_gat_bwd --workload reddit_gat_bwd --steps 6 --no-e2e --no-cpu-baseline
TLP_HOT=0.5 b reddit_hot05 --steps 6 --no-e2e --no-cpu-baseline
b cora --workload cora --steps 20 --no-e2e --no-cpu-baseline
b cora_cg --workload cora --steps 20 --no-e2e --no-cpu-baseline --cuda-graph
b pubmed --workload pubmed --steps 20 --no-e2e --no-cpu-baseline
b pubmed_cg --workload pubmed --steps 20 --no-e2e --no-cpu-baseline --cuda-graph
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s6/gatb_launches.csv \
    python bench.py --workload reddit_gat_bwd --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
