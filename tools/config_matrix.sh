# Every BASELINE-shaped single-GPU config through bench.py with the default (auto) paths.
set -x
o=${1:-gpurun_out/matrix}; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
B="timeout 900 python bench.py --cpu-seconds 2 --e2e-steps 2"
$B --workload tiny > $o/tiny.json 2> $o/tiny.err
for c in 0.02 0.05 0.1; do $B --workload dlr_criteo@0.15 --cache-ratio $c > $o/dlr_c$c.json 2> $o/dlr_c$c.err; done
for c in 0.05 0.1 0.2 0.3 1.0; do $B --cache-ratio $c > $o/pa_c$c.json 2> $o/pa_c$c.err; done
for c in 0.1 1.0; do $B --workload gnn_mag@0.15 --cache-ratio $c > $o/mag_c$c.json 2> $o/mag_c$c.err; done
python tools/matrix_table.py $o > $o/matrix.md
cat $o/matrix.md
