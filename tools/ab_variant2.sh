# warp->node mapping A/B: interleaved (default) vs contiguous (PL_VARIANT=2) at the bench point
export GAINS=0.22344,1.14693,0.07856
for vv in 0 2; do
  echo "== PL_VARIANT=$vv" >> gpurun_out/ab_v2.txt
  PL_VARIANT=$vv python tools/lateness_scan.py 1572 2804 3121 12132 15,16 2 >> gpurun_out/ab_v2.txt 2>&1
  PL_VARIANT=$vv python tools/step_breakdown.py 15 1572 2804 3121 12132 348 5789 4371 30346 1 >> gpurun_out/ab_v2.txt 2>&1
  PL_VARIANT=$vv python tools/s3_worst.py >> gpurun_out/ab_v2.txt 2>&1
done
