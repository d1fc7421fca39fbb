#!/bin/bash
# Build the phase-probe variant of the library (debug only) next to the real one.
cd "$(dirname "$0")/.."
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Xcompiler -fPIC -shared -DSPBLA_PROBE -I include \
  paper_conf_ipps_orachevkkg21_b200/csrc/*.cu -o paper_conf_ipps_orachevkkg21_b200/libspbla_b200_probe.so && echo probe built
