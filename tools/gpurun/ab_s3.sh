# A/B of S3 extension variants on the GPU box: in-tree build vs _variants/$1.so
P="15 1572 2804 3121 12132 348 5789 4371 30346 1"
for v in base "$@"; do
  if [ $v = base ]; then L=""; else L="_variants/$v.so"; fi
  echo "== $v" >> gpurun_out/ab_s3.txt
  PLGPU_LIB=$L python tools/s3_worst.py >> gpurun_out/ab_s3.txt 2>&1
  PLGPU_LIB=$L python tools/step_breakdown.py $P >> gpurun_out/ab_s3.txt 2>&1
done
