mkdir -p gpurun_out/s9
export TLP_SYNTH_CACHE=/tmp/tlp_synth
S=gpurun_out/s9/summary.txt
b() {  # <tag> <bench args...>
  t=$1; shift
  python bench.py "$@" > gpurun_out/s9/$t.json 2> gpurun_out/s9/$t.err
  python -c "import json;d=json.load(open('gpurun_out/s9/$t.json'));print('$t', d['value'], d['ms_per_step'], {k:v['ms_mean'] for k,v in d['ops'].items()}, d['clocks']['sm_mhz'])" >> $S 2>&1
}
b base --steps 5 --no-e2e --no-cpu-baseline
for v in U4B2 U2B4; do
  TLP_LIB_PATH=$PWD/paper_conf_hpdc_fujh22_b200/libtlp_$v.so b $v --steps 5 --no-e2e --no-cpu-baseline
done
TLP_GATHER=async TLP_PANEL=128 b async128 --steps 5 --no-e2e --no-cpu-baseline
b base2 --steps 5 --no-e2e --no-cpu-baseline
TLP_LIB_PATH=$PWD/paper_conf_hpdc_fujh22_b200/libtlp_U4B2.so timeout 600 python -m pytest tests -x -q -m gpu -k "reddit or parity" > gpurun_out/s9/pytest_U4B2.log 2>&1
timeout 600 python -m pytest tests -x -q -m gpu -k "projection" > gpurun_out/s9/pytest_proj.log 2>&1
