# ncu --set full of the emitting join over D' chunk sub-ranges of C5 (SJ_DEBUG_VRANGE)
mkdir -p gpurun_out/prof
for r in ${RANGES:-100000,240173 15000,100000 0,15000}; do
  tag=$(echo $r | tr , _)
  SJ_DEBUG_VRANGE=$r timeout 600 ncu --set full --clock-control none --import-source on -k regex:join_kernel -s 2 -c 1 -o gpurun_out/prof/c5_r$tag python tools/step.py c5 2 > gpurun_out/prof/ncu_r$tag.log 2>&1
  tail -1 gpurun_out/prof/ncu_r$tag.log
  SJ_DEBUG_VRANGE=$r python tools/step.py c5 3 2>&1 | tail -1
done
