# Two-phase kernel with peer roles at small / medium batches (fake peers), back-to-back device
# time per extract (tools/host_overhead.py) under variants of the local / host paths.
o=${1:-gpurun_out/fsmall}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
for v in "X=0" "UGACHE_LOCAL_BULK=1" "UGACHE_WALK_KEYS_PER_SM=1000000000000" "UGACHE_INLINE=3" "UGACHE_PREORDER=0"; do
  t=$(echo $v | tr ' =' '__')
  env $v timeout 600 python tools/host_overhead.py --gpus 2 4 8 --batch-n 2000 20000 100000 500000 > $o/$t.jsonl 2> $o/$t.err
  echo "== $v"; python -c "
import json
for l in open('$o/$t.jsonl'):
    r = json.loads(l); print(r['G'], r['n'], r['mode'], r['path'], r['device_us'])"
done
