# ncu --set full of the single pass (register path, sparse host) and random dispatch on the
# same DLR@0.15 c = 20 % batches (the config where random dispatch is 8 % faster).
o=${1:-gpurun_out/dlrk3}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
for k in stream_extract random_dispatch; do
  timeout 1200 ncu --set full --import-source on --clock-control none -k regex:$k -s 4 -c 2 \
    -o $o/dlr_$k -f python bench.py --workload dlr_criteo@0.15 --cache-ratio 0.2 --steps 3 --warmup 3 --no-calibrate \
    --cpu-seconds 0.5 --no-host-tier > $o/ncu_$k.log 2>&1; echo "ncu $k rc $?"
  ncu -i $o/dlr_$k.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,smsp__inst_executed.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum,sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread > $o/raw_$k.csv 2>&1
  ncu -i $o/dlr_$k.ncu-rep --page details --csv > $o/details_$k.csv 2>&1
  cut -d, -f5,12- $o/raw_$k.csv | tail -2
done
