set -x
o=gpurun_out/r1zb; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
B="timeout 600 python bench.py --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra --stream on"
for pf in 0 1; do
for k in 1 2; do
  UGACHE_STREAM_PREFETCH=$pf UGACHE_STREAM_K=$k $B --workload dlr_criteo@0.15 > $o/dlr0.1_k${k}_p$pf.json 2>/dev/null
  UGACHE_STREAM_PREFETCH=$pf UGACHE_STREAM_K=$k $B --cache-ratio 1.0 > $o/pa100_k${k}_p$pf.json 2>/dev/null
done
done
for f in $o/*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1], round(d["ms_per_step"],4), round(d["kernel_ms"]["factored_gather"],4))
except Exception as e: print(sys.argv[1], "ERR", e)
PY
done
