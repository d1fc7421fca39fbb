#!/bin/bash
# Build variant libraries with overridden hash-bin configs (rowsort.cu HBIN *_CFG macros).
# usage: tools/sweep_build.sh "name1|H1_CFG=a,b,..;H3_CFG=..." ...   (';'-separated defines)
cd "$(dirname "$0")/.."
V=paper_conf_ipps_orachevkkg21_b200/variants; rm -rf $V; mkdir -p $V
for spec in "$@"; do
  name=${spec%%|*}; defs=${spec#*|}
  : > $V/cfg_$name.h
  IFS=';' read -ra DS <<< "$defs"
  for d in "${DS[@]}"; do [ -n "$d" ] && echo "#define ${d%%=*} ${d#*=}" >> $V/cfg_$name.h; done
  ( nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -Xcompiler -O2 -shared -I include \
      -include $V/cfg_$name.h paper_conf_ipps_orachevkkg21_b200/csrc/*.cu -o $V/libspbla_$name.so 2>&1 | grep -E "error" ; echo "built $name" ) &
done
wait
ls $V
