# Round evidence: bench line, ncu launch list, ncu --set full of k_agg launches.
# usage: bash scripts/evidence.sh <round tag> <part: a|b>
R=${1:-r01}
P=${2:-a}
mkdir -p gpurun_out/$R
prof() {  # <regex> <name> <workload>
  ncu --kernel-name-base mangled --set full --clock-control none --import-source on \
      -k "regex:$1" -s 3 -c 1 -o gpurun_out/$R/$2 -f \
      python bench.py --workload $3 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/$R/$2.log 2>&1
}
if [ "$P" = "a" ]; then
  python bench.py > gpurun_out/$R/bench.json 2> gpurun_out/$R/bench.err
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/$R/launches.csv \
      python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
  prof "_ZN3tlp5k_aggILi4ELi0E" reddit_gcn reddit
  prof "_ZN3tlp5k_aggILi4ELi2E" reddit_gat reddit
else
  prof "_ZN3tlp5k_aggILi4ELi1E" reddit_gin reddit
  prof "_ZN3tlp5k_agg" products_gat products
fi
ls -la gpurun_out/$R
