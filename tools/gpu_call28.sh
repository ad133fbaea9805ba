set -x
o=gpurun_out/r1ze; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 300 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "single_pass or stream_auto or timing or fused_and_split or tiny or ragged" > $o/pytest_new.txt 2>&1; echo "rc $?" >> $o/pytest_new.txt
tail -3 $o/pytest_new.txt
grep -q "rc 0" $o/pytest_new.txt || exit 1
timeout 600 python bench.py --workload tiny > $o/bench_tiny.json 2> $o/bench_tiny.err
timeout 600 python bench.py --workload dlr_criteo@0.15 --no-verify --cpu-seconds 1 --e2e-steps 1 > $o/bench_dlr.json 2> $o/bench_dlr.err
for f in $o/bench*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1], round(d["ms_per_step"],4), d.get("kernel_ms"), d.get("fem_ablation"), d.get("parity"))
except Exception as e: print(sys.argv[1], "ERR", e)
PY
done
