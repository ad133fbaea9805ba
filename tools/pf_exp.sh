# Single-pass locate pipeline (UGACHE_STREAM_PREFETCH 0 / 1 / 2): parity tests, then the
# all-local gnn_pa batch (c = 100 %) and DLR@0.15 (c = 10 %), two alternating runs each.
o=${1:-gpurun_out/pf}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "locate_pipeline" > $o/pytest.txt 2>&1; echo "pytest rc $?" >> $o/pytest.txt
for rep in 1 2; do
  for pf in 0 2 1; do
    UGACHE_STREAM_PREFETCH=$pf timeout 300 python bench.py --cache-ratio 1.0 --no-calibrate --cpu-seconds 0.5 > $o/pa100_pf${pf}_r$rep.json 2> $o/pa100_pf${pf}_r$rep.err
    UGACHE_STREAM_PREFETCH=$pf timeout 300 python bench.py --workload dlr_criteo@0.15 --cache-ratio 0.1 --no-calibrate --cpu-seconds 0.5 > $o/dlr_pf${pf}_r$rep.json 2> $o/dlr_pf${pf}_r$rep.err
  done
done
python - $o <<'PY'
import json, sys, glob, os
for f in sorted(glob.glob(sys.argv[1] + "/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(os.path.basename(f), round(d["ms_per_step"], 4), d["cold_l2"]["ms_per_step"].__round__(4), d["roofline"]["bound"], round(d["roofline"]["frac"], 3), d.get("parity"))
    except Exception as e:
        print(f, "ERR", e)
PY
