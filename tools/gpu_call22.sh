set -x
o=gpurun_out/r1y; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
B="timeout 600 python bench.py --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra"
$B --stream on > $o/pa10_stream.json 2>/dev/null
$B --stream on --inline none > $o/pa10_stream_q.json 2>/dev/null
UGACHE_HOST_WARPS=16 $B --stream on --inline none --host-sms 24 > $o/pa10_stream_q24.json 2>/dev/null
$B --stream off > $o/pa10_off.json 2>/dev/null
$B --cache-ratio 0.3 --stream on > $o/pa30_stream.json 2>/dev/null
$B --cache-ratio 0.3 --stream off > $o/pa30_off.json 2>/dev/null
for f in $o/*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1], round(d["ms_per_step"],4), d["roofline"]["path"], round(d["roofline"]["frac"],3))
except Exception as e: print(sys.argv[1], "ERR", e)
PY
done
