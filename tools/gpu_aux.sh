#!/bin/bash
# Measurement lines of the other BASELINE rows: configs[2] (EWiseAdd + Kronecker), configs[3] (closure).
cd "$(dirname "$0")/.."
O=gpurun_out/aux; mkdir -p $O
for wl in ewise_kron closure18; do
  timeout 600 python bench.py --workload $wl --steps 5 > $O/bench_$wl.json 2> $O/bench_$wl.err; cut -c1-400 $O/bench_$wl.json; tail -2 $O/bench_$wl.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_ewise_kron.csv python bench.py --workload ewise_kron --steps 1 --warmup 3 > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k "regex:merge_write|kron_cols" -s 6 -c 2 -o $O/top_aux -f python bench.py --workload ewise_kron --steps 1 --warmup 3 > $O/ncu_aux.log 2>&1
ls -la $O
