#!/bin/bash
# round-2 measurement session on one B200 (run under gpurun): bench lines, ncu launch list and
# the --set full capture of the search kernel for profiles/ 
set -x
mkdir -p gpurun_out
python bench.py --steps 20 --warmup 5 > gpurun_out/r2_bench_c2.json 2> gpurun_out/r2_bench_c2.err
python bench.py --config 5 --steps 5 --warmup 3 > gpurun_out/r2_bench_c5.json 2> gpurun_out/r2_bench_c5.err
python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r2_bench_ref.json 2> gpurun_out/r2_bench_ref.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2_launches.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --no-extra > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_lane_search_c -s 3 -c 1 -o gpurun_out/r2_search_c2 \
    python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu --no-extra > /dev/null 2>&1
ls -la gpurun_out
