#!/bin/bash
# Round-2 evidence capture on the GPU box (repo root): ncu launch lists with DRAM bytes (C3, C4,
# C5) -> profiles/traffic_r02.json (per-kernel bytes per launch, bytes per detect), bench lines
# for every config, compute-sanitizer runs on small traces.
set -u
tag=${1:-r02l}
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
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python profiles/sanitize_driver.py \
    > gpurun_out/${tag}_sanitize_${tool}.log 2>&1
  echo "sanitizer $tool rc=$?"
done
