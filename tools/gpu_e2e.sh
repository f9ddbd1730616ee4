# e2e (host buffers) A/B: default vs no L2 window, twice each; + sort1024 device A/B
for i in 1 2; do for v in default nowin; do
  if [ $v = default ]; then unset HARMONIA_LIB; else export HARMONIA_LIB=gpurun_variants/$v.so; fi
  timeout 300 python bench.py --no-cpu --steps 10 --e2e-steps 10 2>/dev/null | python -c "
import sys,json
d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$v', round(d['value'],2), 'e2e', round(d['e2e']['value'],3))"
done; done
unset HARMONIA_LIB
bash tools/ab_psa.sh 2>/dev/null; bash tools/ab_psa.sh --config 3 2>/dev/null
