#!/bin/bash
# Time experimental libsj variants (exp/libsj_*.so, tools/variant_build.sh) on the GPU box.
# usage: variant_run.sh "cfg1 cfg2 ..." [steps]   (CHECK=1: parity vs the oracle first)
cfgs=${1:-"c4k32 c3k64 c5"}; steps=${2:-4}
for lib in exp/libsj_*.so; do
  if [ -n "$CHECK" ]; then echo "== check $lib"; SJ_LIB_PATH=$lib timeout 600 python tools/variant_check.py 2>&1 | tail -${CHECK_TAIL:-3}; fi
  for c in $cfgs; do
    echo "== $lib $c"
    SJ_LIB_PATH=$lib timeout 300 python tools/step.py $c $steps 2>&1 | tail -2
  done
done
