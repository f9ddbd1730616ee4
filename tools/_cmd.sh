python bench.py > gpurun_out/r1f_bench_c2.json 2> gpurun_out/r1f_bench_c2.err
python bench.py --config 3 > gpurun_out/r1f_bench_c3_zipf.json 2>&1
python bench.py --config 3 --dist uniform > gpurun_out/r1f_bench_c3_uniform.json 2>&1
python bench.py --config 4 > gpurun_out/r1f_bench_c4.json 2>&1
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r1f_bench_ref_c2.json 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_r1f.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_lane_search_c|k_psa2" -c 5 -o gpurun_out/prof_r1f python tools/prof_search.py --calls 1 > gpurun_out/ncu_full.log 2>&1
for f in gpurun_out/r1f_bench_*.json; do echo $f; tail -c 400 $f; echo; done
