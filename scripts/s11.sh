mkdir -p gpurun_out/s11
export TLP_SYNTH_CACHE=/tmp/tlp_synth
S=gpurun_out/s11/summary.txt
b() {  # <tag> <bench args...>
  t=$1; shift
  python bench.py "$@" > gpurun_out/s11/$t.json 2> gpurun_out/s11/$t.err
  python -c "import json;d=json.load(open('gpurun_out/s11/$t.json'));print('$t', d['value'], d['ms_per_step'], {k:v['ms_mean'] for k,v in d['ops'].items()}, d['clocks']['sm_mhz'])" >> $S 2>&1
}
timeout 600 python -m pytest tests -x -q -m gpu -k "narrow or projection or gat_backward" > gpurun_out/s11/pytest.log 2>&1; echo "rc $?" >> gpurun_out/s11/pytest.log
b base --steps 5 --no-e2e --no-cpu-baseline
for m in 112 96 80 72; do TLP_PANEL=$m b p$m --steps 5 --no-e2e --no-cpu-baseline; done
b base2 --steps 5 --no-e2e --no-cpu-baseline
TLP_PANEL=96 b gatb96 --workload reddit_gat_bwd --steps 5 --no-e2e --no-cpu-baseline
b gatb --workload reddit_gat_bwd --steps 5 --no-e2e --no-cpu-baseline
