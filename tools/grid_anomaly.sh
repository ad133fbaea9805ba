# Two slow UGache points of the placement grid (sparse host bucket, peers queued, fused path):
# phase stamps under the default and with pre-ordering / ordering / single-pass variants.
o=${1:-gpurun_out/anom}; mkdir -p $o
python __graft_entry__.py > /dev/null 2>&1
run() {  # name alpha c G [env...]
  local n=$1 a=$2 c=$3 g=$4; shift 4
  env "$@" timeout 300 python tools/placement_grid.py --alphas $a --cache-ratios $c --gpus $g --policies ugache --phases --out $o/$n.jsonl > /dev/null 2> $o/$n.err
  python -c "import json,sys; r=json.loads(open('$o/$n.jsonl').readlines()[-1]); print('$n', [round(x,3) for x in r['ms']], r.get('phases_ms'))"
}
for p in a:1.0:0.2:8 b:1.4:0.5:2; do
  IFS=: read n a c g <<< "$p"
  run ${n}_default $a $c $g
  run ${n}_nopreorder $a $c $g UGACHE_PREORDER=0
  run ${n}_sort_min_1e8 $a $c $g UGACHE_HOST_SORT_MIN=100000000
  run ${n}_sort_min_1 $a $c $g UGACHE_HOST_SORT_MIN=1
  run ${n}_seg1 $a $c $g UGACHE_HOST_SEGMENTS=1
done
