#!/bin/bash
# Measurement session on one B200 (run under gpurun): ncu launch list of the default bench
# command and --set full captures of its kernels first (profiles/ncu_r2.json, which the bench
# line's roofline reads), then the bench lines and extras (profiles/)
mkdir -p gpurun_out
T=${1:-r2e}
LSU=l1tex__data_pipe_lsu_wavefronts.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --no-extra > /dev/null 2>&1
ncu --set full --metrics $LSU --clock-control none --import-source on -k regex:"k_lane_search_c|k_psa2" -s 15 -c 5 \
    -o gpurun_out/${T}_c2 python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu --no-extra > /dev/null 2>&1
ncu --set full --metrics $LSU --clock-control none --import-source on -k regex:"k_lane_search_c|k_psa2|k_l2" -s 40 -c 16 \
    -o gpurun_out/${T}_c4 python tools/prof_search.py --keys 28 --queries 27 --calls 4 > /dev/null 2>&1
python tools/ncu_summary.py --launches gpurun_out/${T}_launches.csv --rep gpurun_out/${T}_c2.ncu-rep \
    --queries-per-launch 67108864 --workload c2_T2^23_F64_Q2^26_uniform --out gpurun_out/${T}_c2 > /dev/null 2>&1
python tools/ncu_summary.py --rep gpurun_out/${T}_c4.ncu-rep --queries-per-launch 134217728 \
    --workload c4_T2^28_F64_Q2^27_uniform_replicated_n1 --out gpurun_out/${T}_c4 > /dev/null 2>&1
rm -f gpurun_out/${T}_c4.ncu-rep
cp profiles/ncu_r2.json gpurun_out/${T}_ncu_r2.json 2>/dev/null
python bench.py --steps 20 --warmup 5 > gpurun_out/${T}_bench_c2.json 2> gpurun_out/${T}_bench_c2.err
python bench.py --config 5 --steps 5 --warmup 3 > gpurun_out/${T}_bench_c5.json 2> gpurun_out/${T}_bench_c5.err
python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/${T}_bench_ref.json 2> gpurun_out/${T}_bench_ref.err
python tools/bench_extras.py --what update,range > gpurun_out/${T}_extras.jsonl 2>&1
python -m pytest tests -m gpu -x -q > gpurun_out/${T}_pytest_gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.txt 2>&1
ls -la gpurun_out | grep $T
du -sh gpurun_out
