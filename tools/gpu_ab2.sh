# A/B of gpurun_variants/*.so over c2, c3 (zipf, uniform, F16, F8), c4; parity of the given variants
T=${1:-ab}; PAR=${2:-}
for cfg in "" "--config 3" "--config 3 --dist uniform" "--config 3 --fanout 16" "--config 3 --fanout 8" "--config 4 --steps 5"; do
  echo "== $cfg"; bash tools/ab_psa.sh $cfg 2>/dev/null
done
for v in $PAR; do
  echo "== parity $v"
  HARMONIA_LIB=gpurun_variants/$v.so timeout 600 python -m pytest tests/test_gpu_search.py -m gpu -x -q 2>&1 | tail -1
done
