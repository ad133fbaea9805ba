set -x
o=gpurun_out/r1zq; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 900 python bench.py > $o/bench.json 2> $o/bench.err
timeout 600 python bench.py --workload dlr_criteo@0.15 --no-verify --cpu-seconds 1 --e2e-steps 1 > $o/bench_dlr.json 2> $o/bench_dlr.err
for f in $o/bench*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1], round(d["ms_per_step"],4), d["host_only"], d["roofline"]["frac"])
except Exception as e: print(sys.argv[1], "ERR", e)
PY
done
tail -3 $o/bench.err
