# A/B round: every gpurun_variants/*.so on c2 and c3 (zipf), parity of selected variants.
#   bash tools/gpu_ab.sh TAG "variant1 variant2 ..."
T=${1:-ab}; PAR=${2:-}
mkdir -p gpurun_out
echo "== c2"; bash tools/ab_psa.sh 2>/dev/null
echo "== c3 zipf"; bash tools/ab_psa.sh --config 3 2>/dev/null
for v in $PAR; do
  echo "== parity $v"
  HARMONIA_LIB=gpurun_variants/$v.so timeout 600 python -m pytest tests/test_gpu_search.py -m gpu -x -q 2>&1 | tail -2
done
