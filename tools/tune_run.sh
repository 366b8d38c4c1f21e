#!/bin/bash
# Run tools/prof_p2p.py against every build/var_*/ library for a set of S values.
cd "$(dirname "$0")/.."
for S in ${SLIST:-32 128 512}; do
  for d in build/var_*/; do
    name=$(basename $d)
    r=$(AFMM_LIB_OVERRIDE=$PWD/$d/libafmm_p2p.so timeout 60 python tools/prof_p2p.py --config ${CONFIG:-C2} --S $S --evals ${EVALS:-10} 2>&1 | grep -oE "int_per_s': np.float64\([0-9.e+]+" | grep -oE "[0-9.e+]+$")
    echo "$name S=$S $r"
  done
done
