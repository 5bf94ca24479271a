#!/bin/bash
# Round-2 final evidence capture on the GPU box (repo root), tag $1:
#   ncu launch lists with DRAM bytes (C5, C4, C3) -> profiles/traffic_r02.json (per-kernel bytes per
#   launch, bytes per detect; read by bench.py), bench lines for C1..C5 (driver recipe), the
#   sync-heavy C2 / C5 variants, the one-rank collective path (C4), streaming sessions (C5),
#   compute-sanitizer on small traces, one ncu --set full of the four streaming kernels.
set -u
tag=${1:-r02f}
for c in C5 C4 C3; do
  w=$(python -c "import tracegen.families as F; print(F.FAMILY_NAMES[${c#C}], F.DEFAULT_N[${c#C}], sep='@')")
  timeout 1500 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --csv --log-file gpurun_out/${tag}_launches_${c}.csv \
    python bench.py --config $c --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/${tag}_ncu_${c}.log 2>&1
  echo "ncu $c rc=$?"
  python profiles/summarize_launches.py gpurun_out/${tag}_launches_${c}.csv "$tag $c launch list" \
    --traffic-json profiles/traffic_r02.json "$w" --detects 4 > gpurun_out/${tag}_launches_${c}_summary.txt
done
cp profiles/traffic_r02.json gpurun_out/traffic_r02.json
for c in C1 C2 C3 C4 C5; do
  timeout 1200 python bench.py --config $c > gpurun_out/${tag}_bench_${c}.json 2> gpurun_out/${tag}_bench_${c}.err
  echo "bench $c rc=$?"
done
for c in C2 C5; do
  timeout 1200 python bench.py --config $c --sync-heavy > gpurun_out/${tag}_bench_${c}_sync_heavy.json 2> gpurun_out/${tag}_bench_${c}_sync_heavy.err
  echo "bench $c sync-heavy rc=$?"
done
timeout 900 python bench.py --config C4 --sharded > gpurun_out/${tag}_bench_C4_sharded.json 2> gpurun_out/${tag}_bench_C4_sharded.err
echo "bench C4 sharded rc=$?"
timeout 900 python bench.py --config C5 --stream-chunks 4 > gpurun_out/${tag}_bench_C5_stream4.json 2> gpurun_out/${tag}_bench_C5_stream4.err
echo "bench C5 stream rc=$?"
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python profiles/sanitize_driver.py \
    > gpurun_out/${tag}_sanitize_${tool}.log 2>&1
  echo "sanitizer $tool rc=$?"
done
timeout 1500 ncu --set full --import-source on --clock-control none --kernel-name-base demangled \
  -k regex:"k_count_fused|k_ingest_sort0|k_onesweep<unsigned long, \(bool\)0|k_check4" -c 6 -o gpurun_out/${tag}_stream \
  python bench.py --config C5 --events 1000000000 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/${tag}_stream.log 2>&1
echo "ncu full rc=$?"
