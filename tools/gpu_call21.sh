set -x
o=gpurun_out/r1x; mkdir -p $o
bash tools/gpu_round_check.sh $o
B="python bench.py --no-verify --e2e-steps 1 --cpu-seconds 1 --no-clocks --steps 3 --warmup 5"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 20 -c 40 --csv --log-file $o/launches_dlr.csv $B --workload dlr_criteo@0.15 > $o/launch_dlr.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 20 -c 40 --csv --log-file $o/launches_pa100.csv $B --cache-ratio 1.0 > $o/launch_pa100.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:stream_extract -s 5 -c 1 -o $o/prof_stream_dlr $B --workload dlr_criteo@0.15 --stream on --no-extra > $o/ncu_dlr.log 2>&1
timeout 600 python bench.py --workload dlr_criteo@0.15 > $o/bench_dlr.json 2> $o/bench_dlr.err
timeout 600 python bench.py --workload dlr_criteo@0.15 --cache-ratio 0.02 > $o/bench_dlr2.json 2> $o/bench_dlr2.err
timeout 600 python bench.py --cache-ratio 1.0 > $o/bench_pa100.json 2> $o/bench_pa100.err
for f in $o/bench*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1], round(d["ms_per_step"],4), d.get("kernel_ms"), d.get("fem_ablation"), d.get("roofline",{}).get("frac"), d.get("source_mix_roofline",{}).get("frac"))
except Exception as e: print(sys.argv[1], "ERR", e)
PY
done
