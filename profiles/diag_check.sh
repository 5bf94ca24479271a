for c in C2 C3 C4; do timeout 300 python profiles/check_stats.py $c; done > gpurun_out/r01s3_check_stats.jsonl 2>&1
timeout 300 python profiles/check_stats.py C5 5e8 >> gpurun_out/r01s3_check_stats.jsonl 2>&1
for s in 0 1 2; do IGD_CHECK_STOP=$s timeout 300 python bench.py --config C5 --events 1000000000 --steps 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('stop$s', json.dumps({k:round(v['ms'],2) for k,v in d['path']['kernels'].items()}))"; done > gpurun_out/r01s3_stop.txt 2>&1
