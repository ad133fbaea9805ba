# Round-end evidence on the final code (one B200): GPU tests, smoke, default bench, reference
# arm, the launch list of the default bench (ncu, cold/serialised), the benched kernel's DRAM /
# PCIe traffic with the host tier (application replay; the launch list runs without the tier:
# under ncu the tier run is OOM-killed, profiles/r2/final/README.md) and an ncu --set full capture of the
# fused kernel on gnn_pa@0.25 (kernel replay; the full-size tier cannot be saved/restored).
o=${1:-gpurun_out/final}; mkdir -p $o
bash tools/gpu_round_check.sh $o
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:"extract|fill" -c 120 --csv \
  --log-file $o/launches_default_notier.csv python bench.py --steps 3 --warmup 3 --no-host-tier > $o/ncu_launches.log 2>&1; echo "launches rc $?"
timeout 1500 ncu --replay-mode application --clock-control none \
  --metrics dram__bytes_read.sum,dram__bytes_write.sum,pcie__read_bytes.sum,pcie__read_bytes.sum.per_second,gpu__time_duration.sum \
  -k regex:fused_extract --launch-skip 2 --launch-count 1 --csv --log-file $o/traffic_fused_tier.csv \
  python tools/profile_capture.py --what traffic > $o/traffic.log 2>&1; echo "traffic rc $?"
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:fused_extract -s 3 -c 1 -o $o/prof_fused_pa025 -f \
  python bench.py --workload gnn_pa@0.25 --steps 3 --warmup 3 --no-extra --no-calibrate --cpu-seconds 0.5 > $o/ncu_full.log 2>&1; echo "full rc $?"
ncu -i $o/prof_fused_pa025.ncu-rep --page details --csv > $o/fused_pa025_details.csv 2>&1
ncu -i $o/prof_fused_pa025.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,pcie__read_bytes.sum,sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread > $o/fused_pa025_raw.csv 2>&1
