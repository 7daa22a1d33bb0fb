# run selected GPU tests: TESTS env (pytest -k expression or paths)
mkdir -p gpurun_out/iter
timeout 1500 python -m pytest ${TPATH:-tests/} -x -q -m gpu ${TK:+-k "$TK"} > gpurun_out/iter/pytest_sel.log 2>&1; tail -15 gpurun_out/iter/pytest_sel.log
