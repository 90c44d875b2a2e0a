mkdir -p gpurun_out/s5
export TLP_SYNTH_CACHE=/tmp/tlp_synth
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/s5/pytest.log 2>&1; echo "rc $?" >> gpurun_out/s5/pytest.log
TLP_TRACE_CREATE=1 python scripts/create_probe.py reddit > gpurun_out/s5/create.log 2>&1
for w in reddit_gat_bwd pubmed_gat_bwd products reddit_bwd; do
  python bench.py --workload $w --steps 5 --no-e2e --cpu-seconds 5 > gpurun_out/s5/b_$w.json 2> gpurun_out/s5/b_$w.err
  python -c "import json;d=json.load(open('gpurun_out/s5/b_$w.json'));print('$w', d['value'],{k:v['ms_mean'] for k,v in d['ops'].items()}, d['clocks']['sm_mhz'], d.get('cpu_baseline'))" >> gpurun_out/s5/summary.txt 2>&1
done
