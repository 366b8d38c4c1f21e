#!/bin/bash
# One GPU call for the round's evidence: GPU tests, the bench line, the ncu launch list of
# the bench command, one `ncu --set full` capture of the C4 P2P kernel
# -> gpurun_out/*_$TAG.*  (compute-sanitizer is closed on the GPU pool this round)
cd "$(dirname "$0")/.."
TAG=${1:-r2}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/tests_$TAG.txt 2>&1
tail -2 gpurun_out/tests_$TAG.txt
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
tail -c 300 gpurun_out/bench_$TAG.json
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_$TAG.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-sweep --no-cpu-baseline \
    --no-stokeslet --no-proxy > /dev/null 2>&1
[ -n "$NO_FULL" ] || timeout 900 ncu --set full --import-source on --clock-control none -k regex:p2p_kernel -s 1 -c 1 \
    -o gpurun_out/p2p_full_C4_$TAG python tools/prof_p2p.py --config C4 --S 256 --evals 2 > /dev/null 2>&1
ls -la gpurun_out | tail -12
