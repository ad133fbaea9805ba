# Small-batch rule (single pass with peers inline up to UGACHE_SMALL_BATCH keys): GPU tests,
# back-to-back device time by batch size (fake peers), tiny at G = 2 (placement grid), and
# the default gnn_pa bench.
o=${1:-gpurun_out/small}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $o/pytest.txt 2>&1; echo "pytest rc $?" >> $o/pytest.txt
timeout 600 python tools/host_overhead.py --gpus 1 2 4 8 --batch-n 2000 8192 20000 32768 50000 100000 > $o/ovh.jsonl 2> $o/ovh.err
UGACHE_SMALL_BATCH=0 timeout 600 python tools/host_overhead.py --gpus 2 8 --batch-n 2000 8192 20000 32768 50000 > $o/ovh_off.jsonl 2> $o/ovh_off.err
timeout 300 python tools/placement_grid.py --workload tiny --alphas 1.2 --cache-ratios 0.1 --gpus 2 --out $o/tiny_grid.jsonl --table $o/tiny_grid.md > /dev/null 2> $o/tiny_grid.err
timeout 300 python bench.py --no-calibrate --cpu-seconds 0.5 > $o/pa10.json 2> $o/pa10.err
python tools/summarize_runs.py $o
python - $o <<'PY'
import json, sys
for f in ("ovh.jsonl", "ovh_off.jsonl"):
    print("==", f)
    for l in open(sys.argv[1] + "/" + f):
        r = json.loads(l); print(r["G"], r["n"], r["mode"], r["path"], r["device_us"])
PY
grep -v "^#\|^$\|^ms" $o/tiny_grid.md
