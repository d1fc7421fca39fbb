#!/bin/bash
# Extra ncu --set full captures (dense bin, H3, upper-bound pass) of one configs[4] MxM -> gpurun_out/ckpt_more/
cd /root/repo
O=gpurun_out/ckpt_more; mkdir -p $O
for kv in "dense:dense_bin_kernel<.int.1024" "H3:hash_bin_kernel<.int.128,..unsigned.int.512," "ub:mxm_ub_kernel"; do
  tag=${kv%%:*}; rx=${kv#*:}
  skip=1; [ "$tag" = ub ] && skip=0
  timeout 900 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k "regex:$rx" -s $skip -c 1 \
     -o $O/top_$tag -f python tools/quick_mxm.py 22 32 0.4 0.2 0.2 5 > $O/ncu_top_$tag.log 2>&1
  tail -1 $O/ncu_top_$tag.log
done
ls $O/*.ncu-rep
