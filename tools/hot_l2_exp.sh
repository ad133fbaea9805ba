# Hot local rows kept in L2 (measured, then removed: the UGACHE_HOT_L2_ROWS / UGACHE_L2_PERSIST_MB
# knobs read slab slots [0, n) with L2 evict_last, optionally with a persisting set-aside):
# gnn_pa c = 100 % and 30 %, two runs each (profiles/r2/hot_l2/).
o=${1:-gpurun_out/hot}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
nvidia-smi --query-gpu=name,clocks.sm --format=csv > $o/smi.txt
for rep in 1 2; do
  for v in 0:0 100000:0 200000:0 100000:64 200000:96 400000:96; do
    h=${v%%:*}; p=${v##*:}
    UGACHE_HOT_L2_ROWS=$h UGACHE_L2_PERSIST_MB=$p timeout 300 python bench.py --cache-ratio 1.0 --no-calibrate --cpu-seconds 0.5 > $o/pa100_h${h}_p${p}_r$rep.json 2> $o/pa100_h${h}_p${p}_r$rep.err
  done
  for v in 0:0 200000:96; do
    h=${v%%:*}; p=${v##*:}
    UGACHE_HOT_L2_ROWS=$h UGACHE_L2_PERSIST_MB=$p timeout 300 python bench.py --cache-ratio 0.3 --no-calibrate --cpu-seconds 0.5 > $o/pa30_h${h}_p${p}_r$rep.json 2> $o/pa30_h${h}_p${p}_r$rep.err
  done
done
python tools/summarize_runs.py $o
