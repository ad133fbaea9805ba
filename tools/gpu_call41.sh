set -x
o=gpurun_out/r1zw; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
UGACHE_ROW_EVICT_FIRST=1 timeout 300 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "single_pass_parity or fused_and_split or row_sizes" > $o/pytest_new.txt 2>&1; echo "rc $?" >> $o/pytest_new.txt
tail -2 $o/pytest_new.txt
grep -q "rc 0" $o/pytest_new.txt || exit 1
B="timeout 600 python bench.py --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra"
for ef in 0 1; do
  UGACHE_ROW_EVICT_FIRST=$ef $B > $o/pa10_ef$ef.json 2>/dev/null
  UGACHE_ROW_EVICT_FIRST=$ef $B --cache-ratio 0.3 > $o/pa30_ef$ef.json 2>/dev/null
  UGACHE_ROW_EVICT_FIRST=$ef $B --workload dlr_criteo@0.15 > $o/dlr_ef$ef.json 2>/dev/null
  UGACHE_ROW_EVICT_FIRST=$ef $B --cache-ratio 1.0 > $o/pa100_ef$ef.json 2>/dev/null
done
for f in $o/*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1].split('/')[-1], round(d["ms_per_step"],4), "throughput", round(d["throughput_mode"]["ms_per_batch"],4))
except Exception as e: print(sys.argv[1], "ERR", e)
PY
done
