mkdir -p gpurun_out/s10
export TLP_SYNTH_CACHE=/tmp/tlp_synth
S=gpurun_out/s10/summary.txt
b() {  # <tag> <bench args...>
  t=$1; shift
  python bench.py "$@" > gpurun_out/s10/$t.json 2> gpurun_out/s10/$t.err
  python -c "import json;d=json.load(open('gpurun_out/s10/$t.json'));print('$t', d['value'], d['ms_per_step'], {k:v['ms_mean'] for k,v in d['ops'].items()}, d['clocks']['sm_mhz'])" >> $S 2>&1
}
b base --steps 5 --no-e2e --no-cpu-baseline
b sage --workload reddit_sage --steps 5 --no-e2e --no-cpu-baseline
TLP_PANEL=64 b pair64 --steps 5 --no-e2e --no-cpu-baseline
b base2 --steps 5 --no-e2e --no-cpu-baseline
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/s10/pytest.log 2>&1; echo "rc $?" >> gpurun_out/s10/pytest.log
