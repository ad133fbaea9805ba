# ncu --set full of the single pass (K3) and random dispatch on the same batch: gnn_pa@0.25,
# G = 1, c = 50 %, 100K keys (4.2 % sparse host rows) -- K3 measured 1.5x slower here.
o=${1:-gpurun_out/k3r}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"extract|random_dispatch" -c 8 \
  -o $o/k3r -f python tools/placement_grid.py --policies ugache --alphas 1.2 --cache-ratios 0.5 --gpus 1 \
  --batch-n 100000 --random --steps 1 > $o/ncu.log 2>&1
echo "ncu rc $?"
ncu -i $o/k3r.ncu-rep --page details --csv > $o/details.csv 2>&1
ncu -i $o/k3r.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,pcie__read_bytes.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__average_warp_latency_issue_stalled_long_scoreboard,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum,lts__t_sectors_srcunit_tex_op_read.sum > $o/raw.csv 2>&1
