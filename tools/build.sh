#!/bin/bash
# Rebuild libspbla_b200.so from the repo root; fails loudly.
set -e
cd "$(dirname "$0")/.."
python -c "import __graft_entry__ as g; g.build()" 2>&1 | grep -vE "^/usr/local/cuda/bin/nvcc" | grep -E "error|warning|Error" || true
python -c "import os,sys; sys.path.insert(0,'.'); from paper_conf_ipps_orachevkkg21_b200 import _build as b; sys.exit(1 if b.is_stale() else 0)" && echo "build ok: $(stat -c %y paper_conf_ipps_orachevkkg21_b200/libspbla_b200.so)"
