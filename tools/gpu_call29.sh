set -x
o=gpurun_out/r1zf; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
B="timeout 600 python bench.py --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra"
for hs in 8 12 16 20; do
for hw in 8 16; do
  UGACHE_HOST_WARPS=$hw $B --host-sms $hs > $o/pa10_hs${hs}_hw$hw.json 2>/dev/null
done
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 0 -c 60 --csv --log-file $o/launches_default.csv python bench.py --steps 3 --warmup 3 --no-extra --no-verify --no-clocks --e2e-steps 1 --cpu-seconds 1 > $o/launch_default.log 2>&1
for f in $o/*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1], round(d["ms_per_step"],4), d.get("kernel_ms"))
except Exception as e: print(sys.argv[1], "ERR", e)
PY
done
