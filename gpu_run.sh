python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; tail -2 gpurun_out/gpu_tests.log
python bench.py --steps 10 --sweep "group_size=2;group_size=2,window=8388608;group_size=2,window=4194304;group_size=2,window=33554432" > gpurun_out/sweep12.jsonl 2>&1; cat gpurun_out/sweep12.jsonl
