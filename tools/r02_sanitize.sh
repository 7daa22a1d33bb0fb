mkdir -p gpurun_out/r02/san
S=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck synccheck initcheck; do
  timeout 1500 $S --tool $tool --print-limit 50 --error-exitcode 9 python tools/sanitize_driver.py > gpurun_out/r02/san/$tool.log 2>&1; echo "$tool rc=$?" >> gpurun_out/r02/san/summary.txt
done
timeout 2400 $S --tool racecheck --racecheck-report analysis --print-limit 50 --error-exitcode 9 python tools/sanitize_driver.py small > gpurun_out/r02/san/racecheck.log 2>&1; echo "racecheck rc=$?" >> gpurun_out/r02/san/summary.txt
cat gpurun_out/r02/san/summary.txt; for f in gpurun_out/r02/san/*.log; do echo == $f; tail -6 $f; done
