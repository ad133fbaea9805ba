set -x
o=gpurun_out/r1p; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 300 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "single_pass or stream_auto or fused_and_split or timing" > $o/pytest_new.txt 2>&1; echo "rc $?" >> $o/pytest_new.txt
tail -3 $o/pytest_new.txt
grep -q "rc 0" $o/pytest_new.txt || exit 1
B="timeout 600 python bench.py --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra"
$B --workload dlr_criteo@0.15 --stream on > $o/dlr_on.json 2> $o/dlr_on.err
$B --workload dlr_criteo@0.15 --cache-ratio 0.02 --stream on > $o/dlr2_on.json 2> $o/dlr2_on.err
$B --cache-ratio 1.0 --stream on > $o/pa100_on.json 2> $o/pa100_on.err
$B --cache-ratio 0.3 --stream on > $o/pa30_on.json 2> $o/pa30_on.err
$B --stream on > $o/pa10_on.json 2> $o/pa10_on.err
$B --workload gnn_mag@0.15 --stream on > $o/mag_on.json 2> $o/mag_on.err
$B --workload gnn_mag@0.15 --stream off > $o/mag_off.json 2> $o/mag_off.err
timeout 900 python -m pytest tests -m gpu -x -q > $o/pytest.txt 2>&1; echo "rc $?" >> $o/pytest.txt; tail -3 $o/pytest.txt
for f in $o/*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1], round(d["ms_per_step"],4), d["kernel_ms"], d["per_source_keys"])
except Exception as e: print(sys.argv[1], "ERR", e)
PY
done
