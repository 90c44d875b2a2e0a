mkdir -p gpurun_out/s7
export TLP_SYNTH_CACHE=/tmp/tlp_synth
S=gpurun_out/s7/summary.txt
timeout 900 python -m pytest tests -x -q -m gpu -k "gat_backward or hot_source" > gpurun_out/s7/pytest.log 2>&1; echo "rc $?" >> gpurun_out/s7/pytest.log
b() {  # <tag> <bench args...>
  t=$1; shift
  python bench.py "$@" > gpurun_out/s7/$t.json 2> gpurun_out/s7/$t.err
  python -c "import json;d=json.load(open('gpurun_out/s7/$t.json'));print('$t', d['value'], d['ms_per_step'], {k:v['ms_mean'] for k,v in d['ops'].items()}, d['clocks']['sm_mhz'])" >> $S 2>&1
}
b reddit --steps 6 --no-e2e --no-cpu-baseline
b reddit_bwd --workload reddit_bwd --steps 6 --no-e2e --no-cpu-baseline
b reddit_gat_bwd --workload reddit_gat_bwd --steps 6 --no-e2e --no-cpu-baseline
TLP_PANEL=128 b reddit_gat_bwd128 --workload reddit_gat_bwd --steps 6 --no-e2e --no-cpu-baseline
b products --workload products --steps 6 --no-e2e --no-cpu-baseline
TLP_TRACE_CREATE=1 python scripts/create_probe.py reddit > gpurun_out/s7/create.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s7/gatb_launches.csv \
    python bench.py --workload reddit_gat_bwd --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
