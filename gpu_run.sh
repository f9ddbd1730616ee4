python -m pytest tests/test_gpu_update.py -m gpu -x -q > gpurun_out/gpu_upd.log 2>&1; tail -30 gpurun_out/gpu_upd.log
