for r in 0,240000 0,20000 0,40000 0,70000 70000,240000 100000,240000 150000,240000 200000,240000; do
  echo "range $r"; SJ_DEBUG_VRANGE=$r python tools/step.py c5 2 2>&1 | tail -1
done
