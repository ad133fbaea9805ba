set -x
o=gpurun_out/r1o; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 300 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "single_pass or stream_auto or fused_and_split" > $o/pytest_new.txt 2>&1; echo "rc $?" >> $o/pytest_new.txt
tail -3 $o/pytest_new.txt
grep -q "rc 0" $o/pytest_new.txt || exit 1
timeout 900 python -m pytest tests -m gpu -x -q > $o/pytest.txt 2>&1; echo "rc $?" >> $o/pytest.txt; tail -3 $o/pytest.txt
B="timeout 600 python bench.py --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra"
for st in off on; do
  for inl in host none; do
    $B --workload dlr_criteo@0.15 --stream $st --inline $inl > $o/dlr_${st}_$inl.json 2> $o/dlr_${st}_$inl.err
    $B --workload dlr_criteo@0.15 --cache-ratio 0.02 --stream $st --inline $inl > $o/dlr2_${st}_$inl.json 2> $o/dlr2_${st}_$inl.err
  done
  $B --cache-ratio 1.0 --stream $st > $o/pa100_$st.json 2> $o/pa100_$st.err
  $B --cache-ratio 0.3 --stream $st > $o/pa30_$st.json 2> $o/pa30_$st.err
done
$B --stream auto > $o/pa10_auto.json 2> $o/pa10_auto.err
$B --workload dlr_criteo@0.15 --mode random > $o/dlr_random.json 2> $o/dlr_random.err
$B --workload dlr_criteo@0.15 --cache-ratio 0.02 --mode random > $o/dlr2_random.json 2> $o/dlr2_random.err
for f in $o/*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1], round(d["ms_per_step"],4), d["kernel_ms"], d["per_source_keys"])
except Exception as e: print(sys.argv[1], "ERR", e)
PY
done
