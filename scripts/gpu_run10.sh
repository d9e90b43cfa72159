set -x
mkdir -p gpurun_out
export PHAST_VERBOSE=1
timeout 300 python -m pytest tests/test_gpu.py -k sweep_modes -x -q 2>&1 | tail -6
PHAST_SWEEP=pipe timeout 400 python bench.py --layout wavefront --cache /tmp/c3w.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r12_pipe.json 2> gpurun_out/r12_pipe.err; cat gpurun_out/r12_pipe.json; tail -3 gpurun_out/r12_pipe.err
for k in 16 32; do PHAST_SWEEP=pipe timeout 300 python bench.py --layout wavefront --k $k --cache /tmp/c3w.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r12_pipe_k$k.json 2>/dev/null; cat gpurun_out/r12_pipe_k$k.json; done
PHAST_SWEEP=pipe timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_pipe -s 3 -c 1 -o /tmp/r12_prof python bench.py --layout wavefront --cache /tmp/c3w.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ncu -i /tmp/r12_prof.ncu-rep --page raw --csv > gpurun_out/r12_prof_raw.csv
cp /tmp/r12_prof.ncu-rep gpurun_out/
