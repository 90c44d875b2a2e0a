# usage: bash scripts/prof.sh <lib tag> <workload> <kernel regex> <out name> [skip]
mkdir -p gpurun_out
v=$1; w=$2; k=$3; o=$4; skip=${5:-3}
TLP_LIB_PATH=$PWD/paper_conf_hpdc_fujh22_b200/$v.so ncu --kernel-name-base mangled --set full --clock-control none --import-source on -k "regex:$k" -s $skip -c 1 -o gpurun_out/$o -f python bench.py --workload $w --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/$o.log 2>&1
tail -2 gpurun_out/$o.log
