# All-local gnn_pa (c = 100 %, single pass): L2 evict-first on row reads and the slot nap.
set -x
o=gpurun_out/r2f; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
B="timeout 600 python bench.py --cache-ratio 1.0 --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra"
for rep in 1 2; do
  $B > $o/pa100_base_$rep.json 2> $o/pa100_base_$rep.err
  UGACHE_ROW_EVICT_FIRST=1 $B > $o/pa100_ef_$rep.json 2> $o/pa100_ef_$rep.err
  UGACHE_STREAM_NAP=0 $B > $o/pa100_nap0_$rep.json 2> $o/pa100_nap0_$rep.err
  UGACHE_STREAM_NAP=400 $B > $o/pa100_nap400_$rep.json 2> $o/pa100_nap400_$rep.err
done
