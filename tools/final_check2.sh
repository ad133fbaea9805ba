# Last round check on the final code (after K3r): GPU tests, smoke, default bench, reference
# arm, and the matrix rows K3r changes (tiny, DLR@0.15 c = 2 / 5 / 10 / 20 %).
o=${1:-gpurun_out/final5}; mkdir -p $o
bash tools/gpu_round_check.sh $o
B="timeout 900 python bench.py --cpu-seconds 2 --e2e-steps 2"
mkdir -p $o/matrix
$B --workload tiny > $o/matrix/tiny.json 2> $o/matrix/tiny.err
for c in 0.02 0.05 0.1 0.2; do $B --workload dlr_criteo@0.15 --cache-ratio $c > $o/matrix/dlr_c$c.json 2> $o/matrix/dlr_c$c.err; done
python tools/matrix_table.py $o/matrix > $o/matrix/matrix.md
