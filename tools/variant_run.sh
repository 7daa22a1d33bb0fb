#!/bin/bash
# Time experimental libsj variants (exp/libsj_*.so, tools/variant_build.sh) on the GPU box.
# usage: variant_run.sh "cfg1 cfg2 ..." [steps]
cfgs=${1:-"c4k32 c3k64 c5"}; steps=${2:-4}
for lib in exp/libsj_*.so; do
  for c in $cfgs; do
    echo "== $lib $c"
    SJ_LIB_PATH=$lib timeout 300 python tools/step.py $c $steps 2>&1 | tail -2
  done
done
