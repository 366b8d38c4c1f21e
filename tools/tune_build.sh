#!/bin/bash
# Build kernel-parameter variants of the library into build/var_<name>/ (for tools/tune_run.sh).
set -e
cd "$(dirname "$0")/.."
SRC=paper_conf_ipps_overmanpmm13_b200/csrc
build() {  # name, -D flags...
  local name=$1; shift
  mkdir -p build/var_$name
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC --expt-relaxed-constexpr -I/opt/prime-rl/.venv/lib/python3.12/site-packages/nvidia/nccl/include \
       -Xptxas -v "$@" -shared -o build/var_$name/libafmm_p2p.so $SRC/afmm_p2p.cu $SRC/peak.cu $SRC/tree_build.cu $SRC/step.cu $SRC/balance.cpp $SRC/finegrained.cpp -ldl \
       2> build/var_$name/ptxas.log
  echo "$name: $(grep -A2 'properties for _ZN4afmm10p2p' build/var_$name/ptxas.log | tr '\n' ' ' | grep -oE '[0-9]+ bytes spill stores|Used [0-9]+ registers')"
}
"$@"
