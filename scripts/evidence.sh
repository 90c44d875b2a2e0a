# Round evidence: bench line, ncu launch list, ncu --set full of each k_agg launch.
# usage: bash scripts/evidence.sh <round tag>
set -x
R=${1:-r01}
mkdir -p gpurun_out/$R
python bench.py > gpurun_out/$R/bench.json 2> gpurun_out/$R/bench.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/$R/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
for op in 0 1 2; do
  ncu --kernel-name-base mangled --set full --clock-control none --import-source on \
      -k "regex:_ZN3tlp5k_aggILi4ELi${op}E" -s 3 -c 1 -o gpurun_out/$R/reddit_op$op -f \
      python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/$R/ncu_op$op.log 2>&1
done
ncu --kernel-name-base mangled --set full --clock-control none --import-source on \
    -k "regex:_ZN3tlp5k_agg" -s 3 -c 1 -o gpurun_out/$R/products_gat -f \
    python bench.py --workload products --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/$R/ncu_products.log 2>&1
ls -la gpurun_out/$R
