#!/bin/bash
# ncu --set full captures of the MxM kernels of configs[4] (rmat22_ef32, seed 5):
# each KERNELS entry "tag:regex" is captured once (skip = Build's launch).
cd "$(dirname "$0")/.."
O=gpurun_out/ncu; mkdir -p $O
IFS=";"; for kv in ${KERNELS:-"H5:hash_bin_kernel<.int.512, .unsigned int.2560" "H3:hash_bin_kernel<.int.256, .unsigned int.512," "H1:hash_bin_kernel<.int.128, .unsigned int.128," "ub:mxm_ub_kernel" "w16:warp_bin_kernel<.int.16>"}; do
  tag=${kv%%:*}; rx=${kv#*:}
  skip=1; [ "$tag" = ub ] && skip=0
  timeout 900 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k "regex:$rx" -s $skip -c 1 \
     -o $O/$tag -f python tools/quick_mxm.py 22 32 0.4 0.2 0.2 5 > $O/$tag.log 2>&1
  tail -1 $O/$tag.log
done
ls -la $O
