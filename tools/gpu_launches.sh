# ncu launch list of tools/step.py for CFG (default c5), summarised per kernel
mkdir -p gpurun_out/iter
C=${CFG:-c5}
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/iter/launches_$C.csv python tools/step.py $C 2 > /dev/null 2>&1
LS_W=100 python tools/launch_summary.py gpurun_out/iter/launches_$C.csv 3 2>&1 | head -40
