set -x
python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; tail -2 gpurun_out/gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
python bench.py > gpurun_out/bench_r1.json 2> gpurun_out/bench_r1.err; cat gpurun_out/bench_r1.json; tail -2 gpurun_out/bench_r1.err
python bench.py --impl reference --steps 5 --warmup 1 > gpurun_out/bench_ref_r1.json 2>&1; tail -1 gpurun_out/bench_ref_r1.json | cut -c1-300
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_ntg_search|k_psa2" -s 8 -c 4 -o gpurun_out/prof_r1 python tools/prof_search.py --calls 2 > gpurun_out/ncu_r1.log 2>&1; tail -1 gpurun_out/ncu_r1.log
