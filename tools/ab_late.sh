# node-0 lateness vs tau0 for the in-tree build and each _variants/$v.so
for v in base "$@"; do
  if [ $v = base ]; then L=""; else L="_variants/$v.so"; fi
  echo "== $v" >> gpurun_out/ab_late.txt
  PLGPU_LIB=$L python tools/lateness_scan.py 1572 2804 3121 12132 13,14,15,16 3 >> gpurun_out/ab_late.txt 2>&1
done
