# iteration check: all gpu tests, step timings of the primary configs, GPU timeline of one C5 step
mkdir -p gpurun_out/round
set -x
timeout 1500 python -m pytest tests/ -x -q -m gpu > gpurun_out/round/pytest.log 2>&1; tail -15 gpurun_out/round/pytest.log
for c in ${CFGS:-c5 c2k64 c3k64 c4k32}; do timeout 300 python tools/step.py $c 4 2>&1 | tail -2; done
timeout 300 python tools/timeline.py c5 3 > gpurun_out/round/tl_c5.txt 2>&1; tail -3 gpurun_out/round/tl_c5.txt
