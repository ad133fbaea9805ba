# Re-entry round check on a fresh container: build, GPU tests, smoke, default bench, reference arm, launch list.
set -x
o=gpurun_out/r2a; mkdir -p $o
bash tools/gpu_round_check.sh $o
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $o/launches.csv python bench.py --steps 2 --warmup 3 --no-verify --e2e-steps 1 --cpu-seconds 1 > $o/bench_under_ncu.log 2>&1
