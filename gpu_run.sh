timeout 1200 python -m pytest tests/test_gpu_large.py -m gpu -x -q -k config5 > gpurun_out/gpu_large.log 2>&1; tail -3 gpurun_out/gpu_large.log
