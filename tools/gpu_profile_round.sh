# Round evidence: bench lines (c2 default contract + c3/c4), ncu launch list, ncu --set full of
# one search call's kernels.   bash tools/gpu_profile_round.sh TAG
T=${1:-rX}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 900 python bench.py > gpurun_out/${T}_bench_c2.json 2> gpurun_out/${T}_bench_c2.err
timeout 600 python bench.py --config 3 --no-cpu --steps 20 > gpurun_out/${T}_bench_c3_zipf.json 2>/dev/null
timeout 600 python bench.py --config 3 --dist uniform --no-cpu --steps 20 > gpurun_out/${T}_bench_c3_uniform.json 2>/dev/null
timeout 900 python bench.py --config 4 --no-cpu --steps 10 > gpurun_out/${T}_bench_c4.json 2>/dev/null
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${T}_bench_ref_c2.json 2>/dev/null
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/${T}_launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:'k_(psa2|lane|sort)' -c 5 \
  -o gpurun_out/${T}_full -f python tools/prof_search.py --calls 1 > gpurun_out/${T}_full.log 2>&1
ls -la gpurun_out | tail -12
