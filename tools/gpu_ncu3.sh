#!/bin/bash
# ncu --set full: dense bin of configs[1] MxM (skip Build's fallback launch),
# the upper-bound pass of configs[4]; Kronecker tests + ewise_kron bench.
cd "$(dirname "$0")/.."
O=gpurun_out/ncu3; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "kron" > $O/pytest_kron.txt 2>&1; tail -2 $O/pytest_kron.txt
timeout 300 python bench.py --workload ewise_kron --steps 9 --warmup 5 > $O/bench_ek.json 2>$O/bench_ek.err; cut -c1-900 $O/bench_ek.json
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k "regex:dense_bin_kernel<.int.1024" -s 1 -c 1 \
   -o $O/dense20 -f python tools/quick_mxm.py 20 16 0.45 0.22 0.22 1 > $O/dense20.log 2>&1
tail -1 $O/dense20.log
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k "regex:mxm_ub_kernel" -s 0 -c 1 \
   -o $O/ub22 -f python tools/quick_mxm.py 22 32 0.4 0.2 0.2 5 > $O/ub22.log 2>&1
tail -1 $O/ub22.log
ls -la $O
