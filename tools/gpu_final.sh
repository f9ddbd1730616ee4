# Final round evidence: GPU tests, smoke, bench lines (c2 contract + c3/c4 + modes), ncu.
T=${1:-rX}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_pytest_gpu.log 2>&1; tail -2 gpurun_out/${T}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
bash tools/gpu_profile_round.sh ${T}
timeout 600 python bench.py --mode partitioned --no-cpu --no-e2e --steps 10 > gpurun_out/${T}_bench_c2_partitioned.json 2>/dev/null
timeout 600 python bench.py --mode peer --no-cpu --no-e2e --steps 10 > gpurun_out/${T}_bench_c2_peer.json 2>/dev/null
for m in partitioned peer; do head -c 200 gpurun_out/${T}_bench_c2_$m.json; echo; done
