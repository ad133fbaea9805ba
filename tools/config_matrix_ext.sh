# SURVEY 8(d) variants beyond the default matrix: gnn_pa at alpha 1.4 (c = 5/10/20 %), DLR@0.15
# at c = 20 %, MAG@0.15 at c = 5 / 20 %.
o=${1:-gpurun_out/matrix_ext}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
B="timeout 900 python bench.py --cpu-seconds 2 --e2e-steps 2"
for c in 0.05 0.1 0.2; do $B --alpha 1.4 --cache-ratio $c > $o/pa14_c$c.json 2> $o/pa14_c$c.err; done
$B --workload dlr_criteo@0.15 --cache-ratio 0.2 > $o/dlr_c0.2.json 2> $o/dlr_c0.2.err
for c in 0.05 0.2; do $B --workload gnn_mag@0.15 --cache-ratio $c > $o/mag_c$c.json 2> $o/mag_c$c.err; done
python tools/matrix_table.py $o > $o/matrix.md
cat $o/matrix.md
