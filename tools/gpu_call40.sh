set -x
o=gpurun_out/r1zv; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "host_first_groups or single_pass_parity" > $o/pytest_new.txt 2>&1; echo "rc $?" >> $o/pytest_new.txt
tail -2 $o/pytest_new.txt
grep -q "rc 0" $o/pytest_new.txt || exit 1
B="timeout 600 python bench.py --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra --stream on"
for gr in 0 2 4 8; do
  UGACHE_STREAM_GROUP=$gr $B --workload dlr_criteo@0.15 > $o/dlr0.1_g$gr.json 2>/dev/null
  UGACHE_STREAM_GROUP=$gr $B --workload dlr_criteo@0.15 --cache-ratio 0.02 > $o/dlr0.02_g$gr.json 2>/dev/null
  UGACHE_STREAM_GROUP=$gr $B --cache-ratio 1.0 > $o/pa100_g$gr.json 2>/dev/null
done
for f in $o/*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1].split('/')[-1], round(d["ms_per_step"],4), round(d["kernel_ms"]["factored_gather"],4))
except Exception as e: print(sys.argv[1], "ERR", e)
PY
done
