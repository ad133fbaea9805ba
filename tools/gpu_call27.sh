set -x
o=gpurun_out/r1zd; mkdir -p $o
bash tools/gpu_round_check.sh $o
timeout 600 python bench.py --workload dlr_criteo@0.15 > $o/bench_dlr.json 2> $o/bench_dlr.err
timeout 600 python bench.py --workload dlr_criteo@0.15 --cache-ratio 0.02 > $o/bench_dlr2.json 2> $o/bench_dlr2.err
timeout 600 python bench.py --cache-ratio 1.0 > $o/bench_pa100.json 2> $o/bench_pa100.err
timeout 600 python bench.py --workload tiny > $o/bench_tiny.json 2> $o/bench_tiny.err
for f in $o/bench*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1], round(d["ms_per_step"],4), d.get("kernel_ms"), d.get("fem_ablation"), d.get("roofline",{}).get("frac"), d.get("roofline",{}).get("path"), d.get("source_mix_roofline",{}).get("frac"))
except Exception as e: print(sys.argv[1], "ERR", e)
PY
done
