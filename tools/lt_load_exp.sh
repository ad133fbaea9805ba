# Location-table lookup instruction (measured, then removed: UGACHE_LT_LOAD 0 ld.global.nc,
# 1 ld.global.cg, 2 ld.global.nc.L1::no_allocate): L2 sectors per lookup (ncu, gnn_pa@0.25,
# c = 100 %, single pass) and bench timing (gnn_pa c = 100 % and 10 %); profiles/r2/lt_load/.
o=${1:-gpurun_out/ltl}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
for v in 0 1 2; do
  UGACHE_LT_LOAD=$v timeout 600 ncu --clock-control none -k regex:"stream_extract|fused_extract" -c 3 \
    --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_requests_srcunit_tex_op_read.sum \
    --csv python tools/placement_grid.py --policies ugache --alphas 1.2 --cache-ratios 1.0 --gpus 1 --steps 1 > $o/ncu_v$v.csv 2> $o/ncu_v$v.err
done
for r in 1 2; do
  for v in 0 1 2; do
    UGACHE_LT_LOAD=$v timeout 300 python bench.py --cache-ratio 1.0 --no-calibrate --cpu-seconds 0.5 > $o/pa100_v${v}_r$r.json 2> $o/pa100_v${v}_r$r.err
    UGACHE_LT_LOAD=$v timeout 300 python bench.py --no-calibrate --cpu-seconds 0.5 > $o/pa10_v${v}_r$r.json 2> $o/pa10_v${v}_r$r.err
  done
done
python tools/summarize_runs.py $o
for v in 0 1 2; do echo "== v$v"; grep -v "^==" $o/ncu_v$v.csv | grep extract | cut -d, -f5,12- ; done
