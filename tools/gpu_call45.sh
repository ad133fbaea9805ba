# Host SM group size on the ordered two-phase path at higher cache ratios (fewer host rows).
set -x
o=gpurun_out/r2d; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
for c in 0.3 0.5; do for hs in 6 12 24 36; do
  timeout 600 python bench.py --cache-ratio $c --host-sms $hs --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra > $o/pa_c${c}_hs$hs.json 2> $o/pa_c${c}_hs$hs.err
done; done
