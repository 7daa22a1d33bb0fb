# per-kernel device times (ncu launch list) of tools/step.py for each config
set -x
for CFG in "$@"; do
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${CFG}.csv python tools/step.py $CFG 2 > /dev/null 2>&1
done
