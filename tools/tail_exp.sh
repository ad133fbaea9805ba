# Launch tail without the host-mirror read: back-to-back device time by batch size and the
# role timelines (fake peers), plus the default gnn_pa bench.
o=${1:-gpurun_out/tail}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 600 python tools/host_overhead.py --gpus 1 2 4 8 --batch-n 2000 20000 100000 500000 > $o/ovh.jsonl 2> $o/ovh.err
timeout 900 python -m pytest tests -m gpu -x -q > $o/pytest.txt 2>&1; echo "pytest rc $?" >> $o/pytest.txt
timeout 600 python tools/role_timeline.py --gpus 1 8 --batch-n 2000 100000 --out $o/tl_raw.json > $o/tl.jsonl 2> $o/tl.err
timeout 300 python bench.py --workload tiny --no-calibrate --cpu-seconds 0.5 > $o/tiny.json 2> $o/tiny.err
timeout 300 python bench.py --no-calibrate --cpu-seconds 0.5 > $o/pa10.json 2> $o/pa10.err
python tools/summarize_runs.py $o
python - $o <<'PY'
import json, sys
for l in open(sys.argv[1] + "/ovh.jsonl"):
    r = json.loads(l); print(r["G"], r["n"], r["mode"], r["path"], r["device_us"])
for l in open(sys.argv[1] + "/tl.jsonl"):
    r = json.loads(l)
    print("G", r["G"], "n", r["n"], "phases", [round(x * 1e3, 1) for x in r["phases_ms"]],
          {k: (v["role_done_us"][1], v["cta_done_us"][1]) for k, v in r["roles"].items()})
PY
