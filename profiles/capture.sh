#!/bin/bash
# Round profile capture (run on the GPU box from the repo root):
#   profiles/capture.sh TAG [CONFIG]
# 1. ncu launch list of the bench command (time + DRAM bytes per launch; single-pass metrics,
#    cold cache, serialised -- shares and bytes, not absolute times) -> gpurun_out/TAG_launches_CFG.csv
# 2. the bench line itself (no profiler) -> gpurun_out/TAG_bench_CFG.json
set -u
tag=$1; cfg=${2:-C5}
timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  --csv --log-file gpurun_out/${tag}_launches_${cfg}.csv \
  python bench.py --config $cfg --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/${tag}_ncu_${cfg}.log 2>&1
echo "ncu rc=$?"
timeout 900 python bench.py --config $cfg > gpurun_out/${tag}_bench_${cfg}.json 2> gpurun_out/${tag}_bench_${cfg}.err
echo "bench rc=$?"
