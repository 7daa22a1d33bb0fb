# selected GPU tests: TK (pytest -k) / TPATH; log under gpurun_out/r02
mkdir -p gpurun_out/r02
timeout ${TT:-2400} python -m pytest ${TPATH:-tests/} -x -q -m gpu ${TK:+-k "$TK"} --durations=15 > gpurun_out/r02/pytest_${TAG:-sel}.log 2>&1; tail -25 gpurun_out/r02/pytest_${TAG:-sel}.log
