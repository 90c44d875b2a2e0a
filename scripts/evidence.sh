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
export TLP_SYNTH_CACHE=/tmp/tlp_synth
if [ "$P" = "a" ]; then
  TLP_TRACE_CREATE=1 python bench.py > gpurun_out/$R/bench.json 2> gpurun_out/$R/bench.err
  # the other configs and context workloads (one line each)
  for w in products pubmed cora rmat24 reddit_f32 products_f32 reddit_sage products_gat4 reddit_bwd reddit_gat_bwd; do
    timeout 900 python bench.py --workload $w --no-cpu-baseline > gpurun_out/$R/bench_$w.json 2> gpurun_out/$R/bench_$w.err
  done
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/$R/launches.csv \
      python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
  prof "_ZN3tlp5k_aggILi4ELi0ELi0E" reddit_gcn reddit
  # GAT on Reddit runs as k_gat_alpha + the streamed-weight sum k_agg<4, 0(GCN), 2(COEF_W), ...>
  prof "_ZN3tlp5k_aggILi4ELi0ELi2E" reddit_gat reddit
  prof "k_gat_alpha" reddit_gat_alpha reddit
else
  prof "_ZN3tlp5k_aggILi4ELi1E" reddit_gin reddit
  prof "_ZN3tlp5k_agg" products_gat products
  prof "_ZN3tlp5k_aggILi4ELi5E" reddit_gatb reddit_gat_bwd
fi
ls -la gpurun_out/$R
if [ "$P" = "b" ] || [ "$P" = "ab" ]; then
  # summarise on the box (gpurun copies back at most 64 MiB): raw pages as CSV,
  # the summary tables, then drop the large .ncu-rep files
  mkdir -p gpurun_out/prof_$R
  for f in gpurun_out/$R/*.ncu-rep; do
    ncu -i "$f" --page raw --csv > gpurun_out/prof_$R/$(basename "$f" .ncu-rep)_raw.csv 2>/dev/null
  done
  PROFILES_OUT=gpurun_out/prof_$R python scripts/make_profiles.py $R > /dev/null 2>&1
  rm -f gpurun_out/$R/*.ncu-rep
fi
