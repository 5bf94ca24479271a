EVARGS="--events 1000000000" bash profiles/run_variants.sh C5 default staged
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_check4 -c 1 -o gpurun_out/r01s3_check4 python bench.py --config C5 --events 500000000 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r01s3_ncu.log 2>&1; echo ncu rc=$?
