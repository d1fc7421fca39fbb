#!/bin/bash
# configs[2] EWiseAdd kernel times for every variant library built by tools/sweep_build.sh.
cd "$(dirname "$0")/.."
O=gpurun_out/sweep_ew; mkdir -p $O; : > $O/summary.txt
for rep in 1 2; do
for so in paper_conf_ipps_orachevkkg21_b200/variants/libspbla_*.so; do
  name=$(basename $so .so); name=${name#libspbla_}
  SPBLA_LIB_PATH=$PWD/$so timeout 300 python bench.py --workload ewise_kron --steps 9 --warmup 5 > $O/$name.json 2> $O/$name.err
  python -c "
import json
d=json.load(open('$O/$name.json'))['ewise']
print('$name', round(d['ms']*1000,1), 'us', {k: round(v*1000,1) for k,v in d['kernel_ms_per_step'].items()}, 'frac', round(d['frac'],3))
" 2>&1 | tee -a $O/summary.txt || tail -3 $O/$name.err
done
done
