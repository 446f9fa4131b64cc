# node-0 lateness vs tau0 for the in-tree build and each _variants/$v.so (GAINS: fixed c2 gains,
# so that variants with node-0 bookkeeping removed can run)
export GAINS=0.22344,1.14693,0.07856
for v in base "$@"; do
  if [ $v = base ]; then L=""; else L="_variants/$v.so"; fi
  echo "== $v" >> gpurun_out/ab_late.txt
  PLGPU_LIB=$L python tools/lateness_scan.py 1572 2804 3121 12132 13,14,15,16 3 >> gpurun_out/ab_late.txt 2>&1
done
