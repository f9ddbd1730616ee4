python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; tail -2 gpurun_out/gpu_tests.log
python bench.py --steps 10 --sweep "group_size=1" 2>&1 | grep sweep
