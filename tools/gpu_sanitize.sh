#!/bin/bash
# compute-sanitizer passes over tools/sanitize.py (every kernel family on small inputs).
# Output: gpurun_out/sanitize_<tool>.txt.   bash tools/gpu_sanitize.sh [tool ...]
export PYTORCH_NO_CUDA_MEMORY_CACHING=1
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in ${@:-memcheck racecheck synccheck initcheck}; do
  small=0; extra=""
  case $tool in
    racecheck) small=1; extra="--racecheck-report hazard" ;;
    initcheck) small=1 ;;
    synccheck) small=1 ;;
  esac
  SANITIZE_SMALL=$small timeout 1500 $CS --tool $tool $extra --print-limit 50 python tools/sanitize.py \
    > gpurun_out/sanitize_$tool.txt 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitize_$tool.txt
  tail -3 gpurun_out/sanitize_$tool.txt
done
