#!/bin/bash
# Kernel-only interactions/s of the in-tree library on C2 for a few S (one GPU).
cd "$(dirname "$0")/.."
for S in ${SLIST:-32 128 512}; do
  timeout 120 python tools/prof_p2p.py --config ${CONFIG:-C2} --S $S --evals 8 2>&1 | python -c "
import sys,re
t=sys.stdin.read(); m=re.search(r\"int_per_s': np.float64\(([0-9.e+]+)\)\",t)
print('S=$S', m.group(1) if m else t[-400:])"
done
