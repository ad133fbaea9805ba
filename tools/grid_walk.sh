# Sparse host bucket with peer roles: input-order walk vs range ordering by batch size
# (UGACHE_WALK_KEYS_PER_SM: 0 = always order, 1e12 = always walk, default 1024), with the
# fused kernel's phase stamps; gnn_pa@0.25, alpha 1.2, c = 20 %, G = 2 / 8 fake peers.
o=${1:-gpurun_out/walk}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
for n in 2000 20000 100000; do
  for w in 0 1024 1000000000000; do
    UGACHE_WALK_KEYS_PER_SM=$w timeout 600 python tools/placement_grid.py --policies ugache --alphas 1.2 --cache-ratios 0.2 --gpus 2 8 --batch-n $n --random --phases --out $o/n${n}_w$w.jsonl > /dev/null 2> $o/n${n}_w$w.err
  done
done
python - $o <<'PY'
import json, glob, sys, statistics
for f in sorted(glob.glob(sys.argv[1] + "/n*.jsonl")):
    for l in open(f):
        r = json.loads(l)
        ph = [p for p in r.get("phases_ms", []) if p]
        med = [round(statistics.median(x), 4) for x in zip(*ph)] if ph else None
        print(f.split("/")[-1], "G", r["G"], "host", round(r["share"]["host"], 4), "ms", round(r["measured_ms"], 4),
              "random", round(r.get("random_dispatch_ms", 0), 4), "phases(loc,ordered,hostdone,lastloc,end)", med,
              "" if r["bit_exact"] else "MISMATCH")
PY
