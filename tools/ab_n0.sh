# A/B of node 0's loop at the bench configuration: in-tree build vs _variants/$v.so
P="15 1572 2804 3121 12132 348 5789 4371 30346"
for v in base "$@"; do
  if [ $v = base ]; then L=""; else L="_variants/$v.so"; fi
  echo "== $v" >> gpurun_out/ab_n0.txt
  PLGPU_LIB=$L python tools/node0_loop.py $P >> gpurun_out/ab_n0.txt 2>&1
done
