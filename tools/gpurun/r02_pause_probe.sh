#!/bin/bash
# Control experiment for the "%globaltimer pause" finding (profiles/r01_globaltimer_pauses.txt):
# the same one-thread probe (tools/probe/gtjump.cu), 10 s each, (a) with no nvidia-smi process and
# no other CUDA context, (b) with `nvidia-smi -lms 100` sampling (the bench's clock sampler),
# (c) with `nvidia-smi -lms 1000`.  Sampler start times are logged to correlate.
set -u
cd "$(dirname "$0")/.."
nvcc -O2 -gencode arch=compute_100a,code=sm_100a -o tools/probe/gtjump tools/probe/gtjump.cu || exit 1
out=gpurun_out/r02_pause_probe.txt
: > $out
for rep in 1 2; do
  echo "== (a) no sampler, rep $rep" >> $out
  ./tools/probe/gtjump 10 >> $out
done
for ms in 100 1000; do
  echo "== (b) nvidia-smi -lms $ms during the probe" >> $out
  t0=$(date +%s.%N)
  nvidia-smi --query-gpu=clocks.sm --format=csv,noheader -lms $ms > gpurun_out/smi_$ms.csv 2>/dev/null &
  pid=$!
  ./tools/probe/gtjump 10 >> $out
  kill $pid; wait $pid 2>/dev/null
  echo "sampler samples: $(wc -l < gpurun_out/smi_$ms.csv) (started ${t0})" >> $out
done
cat $out
