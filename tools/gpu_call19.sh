set -x
o=gpurun_out/r1v; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
B="python bench.py --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra --no-clocks --steps 3 --warmup 5"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:stream_extract -s 5 -c 1 -o $o/prof_stream_pa100 $B --cache-ratio 1.0 --stream on > $o/ncu_pa100.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:stream_extract -s 5 -c 1 -o $o/prof_stream_dlr $B --workload dlr_criteo@0.15 --stream on > $o/ncu_dlr.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 20 -c 40 --csv --log-file $o/launches_dlr.csv $B --workload dlr_criteo@0.15 > $o/launch_dlr.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 20 -c 40 --csv --log-file $o/launches_pa100.csv $B --cache-ratio 1.0 > $o/launch_pa100.log 2>&1
ls -la $o
