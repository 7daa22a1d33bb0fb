mkdir -p gpurun_out/r02/tail
V=240173
SJ_DEBUG_VRANGE=$((V/3)),$V timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:join_kernel<\(int\)2, \(int\)8, \(int\)1" -c 1 -o /tmp/prof_tail python tools/step.py c5 2 > gpurun_out/r02/tail/ncu.log 2>&1
python tools/ncu_summary.py /tmp/prof_tail.ncu-rep > gpurun_out/r02/tail/summary.txt 2>&1
ncu -i /tmp/prof_tail.ncu-rep --page source --csv --print-source sass > gpurun_out/r02/tail/sass.csv 2>/dev/null
cat gpurun_out/r02/tail/summary.txt | head -30; tail -5 gpurun_out/r02/tail/ncu.log
