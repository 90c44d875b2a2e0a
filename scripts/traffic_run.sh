# usage: bash scripts/traffic_run.sh  (on the GPU box) -> gpurun_out/traffic/*
export TLP_SYNTH_CACHE=/tmp/tlp_synth
mkdir -p gpurun_out/traffic
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_sectors.sum,lts__t_sectors_op_write.sum,lts__t_sectors_op_read.sum
for op in gin gcn_both gat; do
  for ld in 604 608; do
    python scripts/traffic_probe.py $op $ld 10 >> gpurun_out/traffic/times.txt 2>&1
    ncu --metrics $M --clock-control none -k regex:k_agg -s 3 -c 1 --csv \
      python scripts/traffic_probe.py $op $ld 1 > gpurun_out/traffic/ncu_${op}_$ld.csv 2>&1
  done
done
TLP_PANEL=0 ncu --metrics $M --clock-control none -k regex:k_agg -s 3 -c 1 --csv \
  python scripts/traffic_probe.py gin 604 1 > gpurun_out/traffic/ncu_gin_604_nopanel.csv 2>&1
