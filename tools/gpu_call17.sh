set -x
o=gpurun_out/r1t; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 300 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "single_pass or stream_auto or timing" > $o/pytest_new.txt 2>&1; echo "rc $?" >> $o/pytest_new.txt
tail -3 $o/pytest_new.txt
grep -q "rc 0" $o/pytest_new.txt || exit 1
B="timeout 600 python bench.py --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra --stream on"
for c in 0.1 0.02; do
  $B --workload dlr_criteo@0.15 --cache-ratio $c > $o/dlr${c}_k2.json 2>/dev/null
  UGACHE_STREAM_K=1 $B --workload dlr_criteo@0.15 --cache-ratio $c > $o/dlr${c}_k1.json 2>/dev/null
  UGACHE_STREAM_STATIC=0 UGACHE_STREAM_K=1 $B --workload dlr_criteo@0.15 --cache-ratio $c > $o/dlr${c}_dyn.json 2>/dev/null
done
$B --cache-ratio 1.0 > $o/pa100_k2.json 2>/dev/null
UGACHE_STREAM_K=1 $B --cache-ratio 1.0 > $o/pa100_k1.json 2>/dev/null
$B --workload gnn_mag@0.15 --cache-ratio 1.0 > $o/mag100_k2.json 2>/dev/null
$B --workload gnn_mag@0.15 --cache-ratio 1.0 --stream off > $o/mag100_off.json 2>/dev/null
$B --workload tiny > $o/tiny_on.json 2>/dev/null
$B --workload tiny --stream off > $o/tiny_off.json 2>/dev/null
timeout 600 python bench.py --no-verify --e2e-steps 1 --cpu-seconds 1 > $o/pa10_default.json 2>/dev/null
timeout 900 python -m pytest tests -m gpu -x -q > $o/pytest.txt 2>&1; echo "rc $?" >> $o/pytest.txt; tail -3 $o/pytest.txt
for f in $o/*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1], round(d["ms_per_step"],4), round(d["kernel_ms"]["factored_gather"],4), d.get("fem_ablation"))
except Exception as e: print(sys.argv[1], "ERR", e)
PY
done
