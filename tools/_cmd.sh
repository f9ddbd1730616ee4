set -x
python -m pytest tests -m gpu -x -q 2>&1 | tail -2
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_r1e.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/launch_bench.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_lane_search_c|k_psa2" -c 5 -o gpurun_out/prof_r1e python tools/prof_search.py --calls 1 > gpurun_out/ncu_full.log 2>&1
tail -2 gpurun_out/ncu_full.log
