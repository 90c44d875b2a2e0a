mkdir -p gpurun_out/s13
export TLP_SYNTH_CACHE=/tmp/tlp_synth
S=gpurun_out/s13/summary.txt
b() {  # <tag> <bench args...>
  t=$1; shift
  TLP_TRACE_CREATE=1 python bench.py "$@" > gpurun_out/s13/$t.json 2> gpurun_out/s13/$t.err
  python -c "import json;d=json.load(open('gpurun_out/s13/$t.json'));print('$t', d['value'], d['ms_per_step'], {k:v['ms_mean'] for k,v in d['ops'].items()}, d['clocks']['sm_mhz'], d['create_ms'])" >> $S 2>&1
}
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/s13/pytest.log 2>&1; echo "rc $?" >> gpurun_out/s13/pytest.log
b reddit --steps 5 --no-e2e --no-cpu-baseline
b rmat --workload rmat24 --steps 3 --no-e2e --no-cpu-baseline
b cora --workload cora --steps 20 --no-e2e --no-cpu-baseline
b bwd --workload reddit_bwd --steps 5 --no-e2e --no-cpu-baseline
b reddit2 --steps 5 --no-e2e --no-cpu-baseline
