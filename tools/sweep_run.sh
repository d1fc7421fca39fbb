#!/bin/bash
# Run bench.py (kernel times) against every variant library built by tools/sweep_build.sh.
cd "$(dirname "$0")/.."
O=gpurun_out/sweep; mkdir -p $O; : > $O/summary.txt
for so in paper_conf_ipps_orachevkkg21_b200/variants/libspbla_*.so; do
  name=$(basename $so .so); name=${name#libspbla_}
  for wl in ${WLS:-rmat22_ef32}; do
    SPBLA_LIB_PATH=$PWD/$so timeout 300 python bench.py --workload $wl --no-cpu-baseline --no-e2e --no-aux --steps 3 > $O/$name.$wl.json 2> $O/$name.$wl.err
    python -c "
import json
d=json.load(open('$O/$name.$wl.json'))
if 'roofline' in d:
    print('$name', '$wl', round(d['ms_per_step'],2),'ms', {k: round(v,2) for k,v in d['roofline']['kernel_ms_per_step'].items() if k[0] in 'Hwd'})
else:
    print('$name', '$wl', round(d['value'],2),'ms', {k: round(v,2) for k,v in d['kernel_ms_per_step'].items() if k[0] in 'Hwd'})
" 2>&1 | tee -a $O/summary.txt || tail -3 $O/$name.$wl.err
  done
done
