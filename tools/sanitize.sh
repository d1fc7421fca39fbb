#!/bin/bash
# compute-sanitizer memcheck + synccheck over the small parity tests (GPU box).
cd "$(dirname "$0")/.."
O=gpurun_out/san; mkdir -p $O
K=${SAN_K:-"mxm_golden or mxm_rmat or ewise or kronecker or closure_golden or duplicate_heavy or rectangular or accumulate"}
timeout 1200 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "$K" > $O/memcheck.txt 2>&1; echo "memcheck rc=$?" >> $O/memcheck.txt
timeout 1200 compute-sanitizer --tool synccheck --print-limit 20 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "$K" > $O/synccheck.txt 2>&1; echo "synccheck rc=$?" >> $O/synccheck.txt
tail -n 4 $O/memcheck.txt; tail -n 4 $O/synccheck.txt
