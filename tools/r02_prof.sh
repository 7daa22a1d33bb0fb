# ncu --set full (+source) of the emitting join launch of the configs in CFGS; summaries + sass csv
mkdir -p gpurun_out/r02/prof_${TAG:-x}
for CFG in ${CFGS:-c5}; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:join_kernel -s 1 -c 1 -o /tmp/prof_${CFG} python tools/step.py $CFG 2 > gpurun_out/r02/prof_${TAG:-x}/ncu_${CFG}.log 2>&1
python tools/ncu_summary.py /tmp/prof_${CFG}.ncu-rep > gpurun_out/r02/prof_${TAG:-x}/${CFG}_summary.txt 2>&1
ncu -i /tmp/prof_${CFG}.ncu-rep --page source --csv --print-source sass > gpurun_out/r02/prof_${TAG:-x}/${CFG}_sass.csv 2> /dev/null
ncu -i /tmp/prof_${CFG}.ncu-rep --page raw --csv > gpurun_out/r02/prof_${TAG:-x}/${CFG}_raw.csv 2>/dev/null
done
cat gpurun_out/r02/prof_${TAG:-x}/*_summary.txt | grep -v "^ *$" | head -60
