python bench.py --config 3 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; tail -c 600 gpurun_out/bench_c3.json; tail -2 gpurun_out/bench_c3.err
python bench.py --config 3 --dist uniform --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_c3u.json 2> gpurun_out/bench_c3u.err; tail -c 300 gpurun_out/bench_c3u.json
python bench.py --config 4 --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err; tail -c 300 gpurun_out/bench_c4.json; tail -2 gpurun_out/bench_c4.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1d.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_lane_search|k_psa2" -s 8 -c 4 -o gpurun_out/prof_r1d python tools/prof_search.py --calls 2 > gpurun_out/ncu_r1d.log 2>&1; tail -1 gpurun_out/ncu_r1d.log
