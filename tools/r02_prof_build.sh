# ncu --set full of every kernel of one C5 build (tools/step.py: sizing handle + 1 step); the
# step's build kernels are summarised (details page) per kernel
mkdir -p gpurun_out/r02/pbuild
timeout 900 ncu --set full --clock-control none --import-source on -o /tmp/prof_build python tools/step.py ${CFG:-c5} 1 > gpurun_out/r02/pbuild/ncu.log 2>&1
ncu -i /tmp/prof_build.ncu-rep --page details --csv > gpurun_out/r02/pbuild/details.csv 2>/dev/null
ncu -i /tmp/prof_build.ncu-rep --page raw --csv > gpurun_out/r02/pbuild/raw.csv 2>/dev/null
ls -la gpurun_out/r02/pbuild
