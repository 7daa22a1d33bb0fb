# iteration check: parity tests (not full size), step timings, launch list of one C5 step
mkdir -p gpurun_out/iter
set -x
timeout 900 python -m pytest tests/ -x -q -m gpu -k "not full_size" > gpurun_out/iter/pytest.log 2>&1; tail -3 gpurun_out/iter/pytest.log
for c in ${CFGS:-c5 c2k64 c3k64 c4k32}; do timeout 300 python tools/step.py $c 4 2>&1 | tail -2; done
if [ -n "$LAUNCHES" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/iter/launches_c5.csv python tools/step.py c5 2 > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/iter/launches_c5.csv 3 2>&1 | head -24
fi
