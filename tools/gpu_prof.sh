# ncu --set full of the emitting join launch (3rd join_kernel launch of tools/step.py) for each config given
set -x
for CFG in "$@"; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:join_kernel -s 2 -c 1 -o gpurun_out/prof_${CFG}_emit python tools/step.py $CFG 2 > gpurun_out/ncu_emit_${CFG}.log 2>&1
tail -2 gpurun_out/ncu_emit_${CFG}.log
done
