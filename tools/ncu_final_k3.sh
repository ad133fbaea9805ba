# ncu --set full of the single-pass kernels on the final code: K3r on DLR@0.15 c = 10 %
# (sparse host, every source inline) and K3 on gnn_pa@0.25 c = 100 % (all-local, TMA slots).
o=${1:-gpurun_out/k3full}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:stream_extract_reg -s 4 -c 1 \
  -o $o/k3r_dlr -f python bench.py --workload dlr_criteo@0.15 --cache-ratio 0.1 --steps 3 --warmup 3 \
  --no-calibrate --no-extra --cpu-seconds 0.5 --no-host-tier > $o/k3r.log 2>&1; echo "k3r rc $?"
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:"stream_extract_kernel" -s 4 -c 1 \
  -o $o/k3_pa100 -f python bench.py --workload gnn_pa@0.25 --cache-ratio 1.0 --steps 3 --warmup 3 \
  --no-calibrate --no-extra --cpu-seconds 0.5 > $o/k3.log 2>&1; echo "k3 rc $?"
for r in k3r_dlr k3_pa100; do
  ncu -i $o/$r.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,pcie__read_bytes.sum,smsp__inst_executed.sum,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active > $o/${r}_raw.csv 2>&1
  ncu -i $o/$r.ncu-rep --page details --csv > $o/${r}_details.csv 2>&1
  cut -d, -f5,12- $o/${r}_raw.csv | tail -1
done
