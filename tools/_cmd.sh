HARMONIA_LIB=gpurun_variants/share.so python -m pytest tests/test_gpu_search.py -x -q 2>&1 | tail -1
bash tools/ab_psa.sh 2>/dev/null
bash tools/ab_psa.sh --config 3 2>/dev/null
bash tools/ab_psa.sh --config 4 2>/dev/null
