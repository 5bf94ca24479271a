#!/bin/bash
# ncu --set full (source-correlated) of the three streaming kernels on C5 at 1e9 events:
#   k_onesweep (access sort pass), k_ingest<0> (pass 0), k_ingest_sort0 (fused write + digit 0)
tag=${1:-r01s3}
timeout 1200 ncu --set full --import-source on --clock-control none \
  -k regex:"k_onesweep<1, unsigned long>|k_ingest<0>|k_ingest_sort0" -c 3 -o gpurun_out/${tag}_stream \
  python bench.py --config C5 --events 1000000000 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/${tag}_stream.log 2>&1
echo ncu rc=$?
