# bench sanity (new fields), join time along the queue (C5), SASS-level profile of the C5 join
mkdir -p gpurun_out/r02/p1
timeout 600 python bench.py --steps 30 --warmup 3 --json-out gpurun_out/r02/p1/bench_c5.jsonl > /dev/null 2> gpurun_out/r02/p1/bench.err; tail -3 gpurun_out/r02/p1/bench.err
timeout 600 python tools/vrange_profile.py c5 12 > gpurun_out/r02/p1/vrange_c5.txt 2>&1
timeout 600 python tools/vrange_profile.py c3k64 12 > gpurun_out/r02/p1/vrange_c3k64.txt 2>&1
cat gpurun_out/r02/p1/vrange_c5.txt
for CFG in c5 c3k64; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:join_kernel -s 1 -c 1 -o /tmp/prof_${CFG} python tools/step.py $CFG 2 > gpurun_out/r02/p1/ncu_${CFG}.log 2>&1
python tools/ncu_summary.py /tmp/prof_${CFG}.ncu-rep > gpurun_out/r02/p1/${CFG}_summary.txt 2>&1
ncu -i /tmp/prof_${CFG}.ncu-rep --page source --csv --print-source sass > gpurun_out/r02/p1/${CFG}_sass.csv 2> /dev/null
ncu -i /tmp/prof_${CFG}.ncu-rep --page raw --csv > gpurun_out/r02/p1/${CFG}_raw.csv 2>/dev/null
done
ls -la gpurun_out/r02/p1
