# A/B the default library against gpurun_variants/*.so on c2 (device-resident bench, no e2e/cpu)
mkdir -p gpurun_out
for v in default $(cd gpurun_variants && ls *.so | sed "s/\.so$//"); do
  if [ $v = default ]; then unset HARMONIA_LIB; else export HARMONIA_LIB=gpurun_variants/$v.so; fi
  python bench.py --no-e2e --no-cpu --steps 20 "$@" > gpurun_out/ab_$v.json 2>/dev/null
  python -c "
import json,sys
d=json.loads(open('gpurun_out/ab_$v.json').read().strip().splitlines()[-1]); kb=d['kernel_breakdown']
print('$v', round(d['value'],2), round(d['ms_per_step'],3), {k:round(x['ms_per_step'],3) for k,x in kb.items()})"
done
