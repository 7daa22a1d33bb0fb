# ncu --set full of the emitting join over D' chunk sub-ranges of C5 (SJ_DEBUG_VRANGE);
# summaries + SASS-level source CSVs are kept, the reports are deleted (gpurun_out cap)
mkdir -p gpurun_out/prof
for r in ${RANGES:-100000,240173 15000,100000 0,15000}; do
  tag=$(echo $r | tr , _)
  SJ_DEBUG_VRANGE=$r timeout 600 ncu --set full --clock-control none --import-source on -k regex:join_kernel -s 2 -c 1 -o /tmp/c5_r$tag python tools/step.py c5 2 > /tmp/ncu_r$tag.log 2>&1
  python tools/ncu_summary.py /tmp/c5_r$tag.ncu-rep > gpurun_out/prof/sum_r$tag.txt 2>&1
  ncu -i /tmp/c5_r$tag.ncu-rep --page source --csv --print-source sass > gpurun_out/prof/sass_r$tag.csv 2>/dev/null
  ncu -i /tmp/c5_r$tag.ncu-rep --page raw --csv > gpurun_out/prof/raw_r$tag.csv 2>/dev/null
  rm -f /tmp/c5_r$tag.ncu-rep
done
ls -la gpurun_out/prof
