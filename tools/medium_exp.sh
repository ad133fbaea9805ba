# Medium batches at G > 1 (fake peers): two-phase (auto) vs single pass with peers queued to
# dedicated SMs (UGACHE_STREAM=1) vs single pass with everything inline (UGACHE_INLINE=3).
o=${1:-gpurun_out/medium}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
for v in "X=0" "UGACHE_STREAM=1" "UGACHE_STREAM=1 UGACHE_INLINE=3"; do
  t=$(echo $v | tr ' =' '__')
  env $v timeout 600 python tools/host_overhead.py --gpus 2 4 8 --batch-n 50000 100000 200000 500000 > $o/$t.jsonl 2> $o/$t.err
  echo "== $v"; python -c "
import json
for l in open('$o/$t.jsonl'):
    r = json.loads(l); print(r['G'], r['n'], r['mode'], r['path'], r['device_us'])"
done
