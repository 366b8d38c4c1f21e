#!/bin/bash
# Round-end evidence (one GPU): GPU tests, bench line, ncu launch list + full capture,
# C5 time loop (plain and load-balanced), strong-scaling proxy.  -> gpurun_out/*_TAG*
cd "$(dirname "$0")/.."
TAG=${1:-r1}
bash tools/measure_all.sh $TAG
timeout 600 python tools/run_c5.py --steps 200 > gpurun_out/c5_timing_$TAG.txt 2>&1
timeout 900 python tools/scaling_proxy.py --config C2 > gpurun_out/scaling_$TAG.txt 2>&1
timeout 900 python tools/scaling_proxy.py --config C3 --worlds 2,4,8 --rebalance 1 >> gpurun_out/scaling_$TAG.txt 2>&1
timeout 900 python tools/scaling_proxy.py --config C4 --worlds 8 --rebalance 1 >> gpurun_out/scaling_$TAG.txt 2>&1
