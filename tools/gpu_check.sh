# Re-entry check: GPU parity suite + c2 bench line.   bash tools/gpu_check.sh TAG
T=${1:-rX}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${T}_smi.txt
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/${T}_pytest_gpu.log 2>&1; tail -3 gpurun_out/${T}_pytest_gpu.log
timeout 600 python bench.py > gpurun_out/${T}_bench_c2.json 2> gpurun_out/${T}_bench_c2.err; cat gpurun_out/${T}_bench_c2.json | head -c 600
echo; bash tools/ab_psa.sh 2>/dev/null
