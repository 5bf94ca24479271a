#!/bin/bash
# ncu --set full (source-correlated) of one access-sort pass (k_onesweep, 12-byte elements) on C5 at 1e9 events
tag=${1:-r02ab}
timeout 1200 ncu --set full --import-source on --clock-control none --kernel-name-base demangled \
  -k regex:"k_onesweep<unsigned long, \(bool\)0" -c 1 -o gpurun_out/${tag}_sort \
  python bench.py --config C5 --events 1000000000 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/${tag}_sort.log 2>&1
echo ncu rc=$?
