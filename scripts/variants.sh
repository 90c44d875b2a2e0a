# usage: bash scripts/variants.sh "tag1 tag2 ..." "workloads"
mkdir -p gpurun_out
V=${1:-"libtlp"}
W=${2:-"reddit"}
for v in $V; do
  for w in $W; do
    TLP_LIB_PATH=$PWD/paper_conf_hpdc_fujh22_b200/$v.so python bench.py --workload $w --steps 8 --no-e2e --no-cpu-baseline > gpurun_out/b_${v}_$w.json 2>gpurun_out/b_${v}_$w.err
    python -c "import json;d=json.load(open('gpurun_out/b_${v}_$w.json'));print('$v $w', d['value'],{k:v['ms_mean'] for k,v in d['ops'].items()})" 2>&1 | tail -1
  done
done
