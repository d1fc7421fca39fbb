#!/bin/bash
# compute-sanitizer memcheck + synccheck + racecheck over the small parity
# tests that cover every bin (GPU box): warp bins and H0-H6 (R-MAT sizes,
# accumulate, rectangular), bitmap/dense (heavy rows, 2^26-column partition
# mode), duplicate-heavy fallback and the closure-step routing, goldens,
# EWiseAdd / Kronecker, closure.
cd "$(dirname "$0")/.."
O=gpurun_out/san; mkdir -p $O
K=${SAN_K:-"mxm_golden or mxm_rmat or ewise or kronecker or closure_golden or duplicate_heavy or rectangular or accumulate or heavy_rows or closure_step or labeled_dag"}
for tool in memcheck synccheck racecheck; do
  timeout 2400 compute-sanitizer --tool $tool --print-limit 20 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "$K" > $O/$tool.txt 2>&1; echo "$tool rc=$?" >> $O/$tool.txt
  tail -n 3 $O/$tool.txt
done
