#!/bin/bash
# Round-2 closing capture at HEAD (repo root), tag $1: ncu launch lists with DRAM bytes (C5, C4, C3)
# -> profiles/traffic_r02.json, driver-recipe bench lines C1..C5 (+ C5 sync-heavy, C4 sharded, C4
# streaming session), one ncu --set full of the six streaming kernels at C5 @ 1e9.  (compute-sanitizer
# is closed on this pool; the r02l / r02m sanitizer logs stand.)
set -u
tag=${1:-r02g}
for c in C5 C4 C3; do
  w=$(python -c "import tracegen.families as F; print(F.FAMILY_NAMES[${c#C}], F.DEFAULT_N[${c#C}], sep='@')")
  timeout 1500 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --csv --log-file gpurun_out/${tag}_launches_${c}.csv \
    python bench.py --config $c --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/${tag}_ncu_${c}.log 2>&1
  echo "ncu $c rc=$?"
  python profiles/summarize_launches.py gpurun_out/${tag}_launches_${c}.csv "$tag $c launch list" \
    --traffic-json profiles/traffic_r02.json "$w" --detects 5 > gpurun_out/${tag}_launches_${c}_summary.txt
done
cp profiles/traffic_r02.json gpurun_out/traffic_r02.json
for c in C1 C2 C3 C4 C5; do
  timeout 1200 python bench.py --config $c > gpurun_out/${tag}_bench_${c}.json 2> gpurun_out/${tag}_bench_${c}.err
  echo "bench $c rc=$?"
done
timeout 1200 python bench.py --config C5 --sync-heavy > gpurun_out/${tag}_bench_C5_sync_heavy.json 2> gpurun_out/${tag}_bench_C5_sync_heavy.err
echo "bench C5 sync-heavy rc=$?"
timeout 900 python bench.py --config C4 --sharded > gpurun_out/${tag}_bench_C4_sharded.json 2> gpurun_out/${tag}_bench_C4_sharded.err
echo "bench C4 sharded rc=$?"
timeout 900 python bench.py --config C4 --stream-chunks 4 > gpurun_out/${tag}_bench_C4_stream4.json 2> gpurun_out/${tag}_bench_C4_stream4.err
echo "bench C4 stream rc=$?"
timeout 1500 ncu --set full --import-source on --clock-control none --kernel-name-base demangled \
  -k regex:"k_count_fused|k_ingest_sort0|k_onesweep<unsigned long, \(bool\)0|k_check4" -c 6 -o gpurun_out/${tag}_stream \
  python bench.py --config C5 --events 1000000000 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/${tag}_stream.log 2>&1
echo "ncu full rc=$?"
