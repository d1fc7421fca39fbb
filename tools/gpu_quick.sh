#!/bin/bash
# Quick GPU iteration: parity tests + bench (both R-MAT workloads) with per-kernel times.
cd "$(dirname "$0")/.."
O=gpurun_out/${QDIR:-quick}; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 400 ${PYTEST_K:+-k "$PYTEST_K"} > $O/pytest.txt 2>&1; tail -2 $O/pytest.txt
for wl in ${WLS:-rmat22_ef32 rmat20_ef16}; do
  timeout 300 python bench.py --workload $wl --no-cpu-baseline --no-e2e --steps 3 > $O/bench_$wl.json 2> $O/bench_$wl.err
  python -c "
import json,sys
d=json.load(open('$O/bench_$wl.json'))
print('$wl', round(d['ms_per_step'],2),'ms', round(d['value'],2), d['unit'], 'peak', round(d['peak_mem_gb'],2),'GB')
print({k: round(v,2) for k,v in d['roofline']['kernel_ms_per_step'].items()})
" 2>&1 | tee -a $O/summary.txt || tail -5 $O/bench_$wl.err
done
