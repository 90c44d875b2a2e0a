mkdir -p gpurun_out/s12
export TLP_SYNTH_CACHE=/tmp/tlp_synth
S=gpurun_out/s12/summary.txt
b() {  # <tag> <bench args...>
  t=$1; shift
  python bench.py "$@" > gpurun_out/s12/$t.json 2> gpurun_out/s12/$t.err
  python -c "import json;d=json.load(open('gpurun_out/s12/$t.json'));print('$t', d['value'], d['ms_per_step'], {k:v['ms_mean'] for k,v in d['ops'].items()}, d['clocks']['sm_mhz'], d['create_ms'])" >> $S 2>&1
}
b products --workload products --steps 6 --no-e2e --no-cpu-baseline
for v in D24B2 D12B4 D8B4; do
  TLP_LIB_PATH=$PWD/paper_conf_hpdc_fujh22_b200/libtlp_$v.so b p_$v --workload products --steps 6 --no-e2e --no-cpu-baseline
done
b rmat --workload rmat24 --steps 3 --no-e2e --no-cpu-baseline
TLP_LIB_PATH=$PWD/paper_conf_hpdc_fujh22_b200/libtlp_D12B4.so b rmat_D12B4 --workload rmat24 --steps 3 --no-e2e --no-cpu-baseline
b products2 --workload products --steps 6 --no-e2e --no-cpu-baseline
b p_gat4 --workload products_gat4 --steps 6 --no-e2e --no-cpu-baseline
TLP_LIB_PATH=$PWD/paper_conf_hpdc_fujh22_b200/libtlp_D12B4.so b p_gat4_D12B4 --workload products_gat4 --steps 6 --no-e2e --no-cpu-baseline
