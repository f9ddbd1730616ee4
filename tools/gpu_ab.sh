#!/bin/bash
for lt in 23 26; do
  AB_ROOT=tools/bin/r1repo PYTHONPATH=tools/bin/r1repo python tools/ab_search.py $lt 26 r1
  python tools/ab_search.py $lt 26 cur
done
python tools/exp_l16.py c4
python -m pytest -x -q tests/test_gpu_psa.py tests/test_gpu_search.py 2>&1 | tail -2
