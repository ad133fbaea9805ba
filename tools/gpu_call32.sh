set -x
o=gpurun_out/r1zu; mkdir -p $o
bash tools/gpu_round_check.sh $o
