# sweep option sets on c2/c3 for the default library and each gpurun_variants/*.so
# usage: bash tools/gpu_sweep.sh "<sweep spec>" [configs...]
spec="$1"; shift
mkdir -p gpurun_out
for c in ${@:-2}; do
for v in default $(ls gpurun_variants 2>/dev/null | grep '\.so$' | sed 's/\.so$//'); do
  if [ $v = default ]; then unset HARMONIA_LIB; else export HARMONIA_LIB=gpurun_variants/$v.so; fi
  python bench.py --config $c --steps 10 --sweep "$spec" 2>/dev/null | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); print('c$c', '$v', {k:v for k,v in d['sweep'].items() if v}, round(d['gqs'],2), {k:round(x,3) for k,x in d['kernels_ms_per_step'].items()})
" | tee -a gpurun_out/sweep.txt
done; done
