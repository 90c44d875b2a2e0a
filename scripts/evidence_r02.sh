# Round-2 evidence on the GPU box: bench lines of every workload, the ncu
# launch list of the default bench step, ncu --set full of the top kernels
# (raw CSV pages only; summarised off-box by scripts/summarize_profiles.py).
# usage: bash scripts/evidence_r02.sh [part: bench|ncu|all]
R=r02; O=gpurun_out/$R; mkdir -p $O
P=${1:-all}
export TLP_SYNTH_CACHE=/tmp/tlp_synth
if [ "$P" = "bench" ] || [ "$P" = "all" ]; then
  TLP_TRACE_CREATE=1 python bench.py > $O/bench.json 2> $O/bench.err
  # short steps get more of them, so the clock sampler sees >= ~10 samples
  for w in rmat24 reddit_sage reddit_bwd reddit_gat_bwd; do
    timeout 900 python bench.py --workload $w --no-cpu-baseline > $O/bench_$w.json 2> $O/bench_$w.err
  done
  for w in products products_gat4 products_f32; do
    timeout 900 python bench.py --workload $w --no-cpu-baseline --steps 60 > $O/bench_$w.json 2> $O/bench_$w.err
  done
  timeout 900 python bench.py --workload reddit_f32 --no-cpu-baseline --steps 200 > $O/bench_reddit_f32.json 2> $O/bench_reddit_f32.err
  for w in cora pubmed; do
    timeout 900 python bench.py --workload $w --no-cpu-baseline --steps 40000 --warmup 100 > $O/bench_$w.json 2> $O/bench_$w.err
  done
  # the multi-rank launcher and the NCCL dist path at world 1 (one GPU per box)
  timeout 900 python bench.py --gpus 1 --spawn --dist --no-cpu-baseline > $O/bench_dist1.json 2> $O/bench_dist1.err
fi
if [ "$P" = "ncu" ] || [ "$P" = "all" ]; then
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv \
      python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
  prof() {  # <name> <kernel regex> <skip> <cmd...>
    n=$1; k=$2; sk=$3; shift 3
    ncu --set full --import-source on --clock-control none -k regex:$k -s $sk -c 1 -o $O/$n -f "$@" > $O/$n.log 2>&1
    ncu -i $O/$n.ncu-rep --page raw --csv > $O/${n}_raw.csv 2>/dev/null
    rm -f $O/$n.ncu-rep
  }
  prof reddit_gcn k_agg 3 python scripts/traffic_probe.py gcn_both 604 1
  prof reddit_gin k_agg 3 python scripts/traffic_probe.py gin 604 1
  prof reddit_gat k_agg 3 python scripts/traffic_probe.py gat 604 1
  prof reddit_gat_alpha k_gat_alpha 3 python scripts/traffic_probe.py gat 604 1
  prof reddit_repack k_repack 3 python scripts/traffic_probe.py gin 604 1
  prof reddit_gat_online k_agg 3 env TLP_GAT=online python scripts/traffic_probe.py gat 604 1
  prof products_gat k_agg 3 python scripts/one_call.py products gat 4
  prof products_gat4 k_agg 3 python scripts/one_call.py products gat4 4
  prof rmat24_gcn k_agg 3 python scripts/one_call.py rmat24 gcn 4
  prof cora_gcn k_rows 3 python scripts/one_call.py cora gcn 4
  prof pubmed_gat k_rows 3 python scripts/one_call.py pubmed gat 4
  prof reddit_outdeg k_out_degree 1 python scripts/create_probe.py reddit
  TLP_TRACE_CREATE=1 python scripts/create_probe.py reddit > $O/create_probe.txt 2>&1
fi
ls -la $O
if [ "$P" = "probes" ] || [ "$P" = "all" ]; then
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tma_probe bench_probe/tma_gather_probe.cu -lcuda > $O/tma_build.log 2>&1
  timeout 300 /tmp/tma_probe > $O/tma_probe.txt 2>&1
  python scripts/host_probe.py > $O/host_probe.txt 2>&1
  (cd scripts && python small_probe2.py > ../$O/small_probe.txt 2>&1)
  (cd scripts && python rows_probe.py > ../$O/rows_probe.txt 2>&1)
fi
