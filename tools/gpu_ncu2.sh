#!/bin/bash
# ncu --set full captures: dense bin on configs[1] (rmat20_ef16) and the
# H3/H5 hash bins on configs[4].  Output: gpurun_out/ncu2/
cd "$(dirname "$0")/.."
O=gpurun_out/ncu2; mkdir -p $O
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k "regex:dense_bin_kernel<1024" -s 0 -c 1 \
   -o $O/dense20 -f python tools/quick_mxm.py 20 16 0.45 0.22 0.22 1 > $O/dense20.log 2>&1
tail -2 $O/dense20.log
for kv in ${KERNELS:-"H5:hash_bin_kernel<.int.512," "H3:hash_bin_kernel<.int.128,"}; do
  tag=${kv%%:*}; rx=${kv#*:}
  timeout 900 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k "regex:$rx" -s 1 -c 1 \
     -o $O/$tag -f python tools/quick_mxm.py 22 32 0.4 0.2 0.2 5 > $O/$tag.log 2>&1
  tail -1 $O/$tag.log
done
ls -la $O
