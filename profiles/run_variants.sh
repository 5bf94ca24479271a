#!/bin/bash
# Benchmark tuning variants of libigd (built into variants/ with -D overrides) on one workload.
# usage: profiles/run_variants.sh C5 name1 name2 ...   (name "default" = the in-tree library;
# "name@VAR=val" runs variant `name` with environment VAR=val; EVARGS adds bench.py arguments)
cfg=$1; shift
for spec in "$@"; do
  v=${spec%%@*}; envs=""; [ "$spec" != "$v" ] && envs=${spec#*@}
  lib=variants/libigd_$v.so; [ "$v" = "default" ] && lib=paper_conf_sosp_kamathb21_b200/libigd.so
  env $envs IGD_LIB=$lib timeout 600 python bench.py --config $cfg --steps 3 ${EVARGS:-} --no-e2e --no-cpu-baseline 2>/dev/null | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$spec', round(d['value'],3), round(d['ms_per_step'],1), d['config']['reports']==d['config']['ledger_reports'], json.dumps({k:round(v['ms'],1) for k,v in d['path']['kernels'].items()}))"
done
