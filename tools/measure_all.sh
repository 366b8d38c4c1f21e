#!/bin/bash
# One GPU call: full GPU test suite, the bench line, the ncu launch list of the
# bench command and one `ncu --set full` capture of the P2P kernel (C2, S=128).
#   gpurun -- 'bash tools/measure_all.sh TAG'   -> gpurun_out/{tests,bench,launches,p2p_full}_TAG.*
cd "$(dirname "$0")/.."
TAG=${1:-r1}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/tests_$TAG.txt 2>&1
tail -3 gpurun_out/tests_$TAG.txt
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
tail -c 600 gpurun_out/bench_$TAG.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-sweep --no-cpu-baseline \
    --no-stokeslet > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:p2p_kernel -s 2 -c 1 \
    -o gpurun_out/p2p_full_$TAG python tools/prof_p2p.py --config C2 --S 128 --evals 3 > /dev/null 2>&1
ls -la gpurun_out | tail -8
