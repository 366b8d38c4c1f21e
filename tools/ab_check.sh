#!/bin/bash
# Parity subset + A/B timing of every build/var_*/ library (one GPU).
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
libs=""
for d in build/var_*/; do
  if [ -n "$NOPARITY" ]; then libs="$libs $d/libafmm_p2p.so"; continue; fi
  r=$(AFMM_LIB_OVERRIDE=$PWD/$d/libafmm_p2p.so timeout 300 python -m pytest tests/test_gpu_p2p.py -x -q \
      -k "c1 or ragged or single or big or determ or momentum or c2_plummer_parity_full" 2>&1 | tail -1)
  echo "$d parity: $r"
  case "$r" in *failed*|*error*) ;; *) libs="$libs $d/libafmm_p2p.so";; esac
done
python tools/ab.py --reps ${REPS:-2} --S ${SLIST:-32,128,512} $libs $EXTRA_LIBS
