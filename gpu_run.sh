python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; tail -2 gpurun_out/gpu_tests.log
python bench.py --steps 10 --sweep "group_size=2;group_size=2,flags=16;group_size=4;group_size=4,flags=16;group_size=8" > gpurun_out/sweep14.jsonl 2>&1; cat gpurun_out/sweep14.jsonl
