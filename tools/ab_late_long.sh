# node-0 lateness at tau0 = 14/15 ns on 1x and 4x the bench stream length, in-tree build vs variants
export GAINS=0.22344,1.14693,0.07856
for v in base "$@"; do
  if [ $v = base ]; then L=""; else L="_variants/$v.so"; fi
  for D in 1048576 4194304; do
    echo "== $v db_len $D" >> gpurun_out/ab_late_long.txt
    PLGPU_LIB=$L python tools/lateness_scan.py 1572 2804 3121 12132 14,15 2 $D >> gpurun_out/ab_late_long.txt 2>&1
  done
done
