# ncu --set full of one emitting join launch per config + per-SASS-instruction source page
mkdir -p gpurun_out/sass
set -x
for CFG in "$@"; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:join_kernel -s 1 -c 1 -o /tmp/prof_${CFG} python tools/step.py $CFG 2 > gpurun_out/sass/ncu_${CFG}.log 2>&1
tail -2 gpurun_out/sass/ncu_${CFG}.log
python tools/ncu_summary.py /tmp/prof_${CFG}.ncu-rep > gpurun_out/sass/${CFG}_summary.txt 2>&1
ncu -i /tmp/prof_${CFG}.ncu-rep --page source --csv --print-source sass > gpurun_out/sass/${CFG}_sass.csv 2> gpurun_out/sass/${CFG}_sass.err
ncu -i /tmp/prof_${CFG}.ncu-rep --page raw --csv > gpurun_out/sass/${CFG}_raw.csv 2>/dev/null
ls -la gpurun_out/sass/
done
