set -x
o=gpurun_out/r1zr; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
UGACHE_LOCAL_SMS=16 timeout 300 python -m pytest tests/test_gpu_extract.py -m gpu -x -q -k "fused_and_split or host_range_ordering or pa_shaped" > $o/pytest_new.txt 2>&1; echo "rc $?" >> $o/pytest_new.txt
tail -2 $o/pytest_new.txt
B="timeout 600 python bench.py --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra"
for ls in 0 96 64 32 16 8; do
  UGACHE_LOCAL_SMS=$ls $B > $o/pa10_ls$ls.json 2>/dev/null
done
for f in $o/*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1], round(d["ms_per_step"],4), round(d["kernel_ms"]["factored_gather"],4))
except Exception as e: print(sys.argv[1], "ERR", e)
PY
done
