# Launch list of the default bench command on the final code (same flags as gpu_call29).
set -x
o=gpurun_out/r2e; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 0 -c 60 --csv --log-file $o/launches_default.csv python bench.py --steps 3 --warmup 3 --no-extra --no-verify --no-clocks --e2e-steps 1 --cpu-seconds 1 > $o/launch_default.log 2>&1
