#!/bin/bash
# ncu --set full (source-correlated) of the four streaming kernels of the fused pipeline on C5 at
# 1e9 events: pass 0 (k_count_fused), the fused write + digit 0 (k_ingest_sort0), one access-sort
# pass (k_onesweep, 12-byte elements) and the check (k_check4).
tag=${1:-r02z}
timeout 1500 ncu --set full --import-source on --clock-control none \
  -k regex:"k_count_fused|k_ingest_sort0|k_onesweep<unsigned long, 0|k_check4" -c 6 -o gpurun_out/${tag}_stream \
  python bench.py --config C5 --events 1000000000 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/${tag}_stream.log 2>&1
echo ncu rc=$?
