#!/bin/bash
# A/B of library variants (tools/bin/*.so, tools/build_variant.py) on one box: c2 and c4 step
# and kernel times.   bash tools/gpu_ab.sh "variant1 variant2 ..."
for v in cur $1; do
  for cfg in c2 c4; do
    if [ "$v" = cur ]; then python tools/exp_l16.py $cfg 2>&1 | grep auto | sed "s/^/$v /";
    else HARMONIA_LIB=tools/bin/$v.so python tools/exp_l16.py $cfg 2>&1 | grep auto | sed "s/^/$v /"; fi
  done
done
