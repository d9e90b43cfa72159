set -x
mkdir -p gpurun_out
export PHAST_VERBOSE=1
timeout 600 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -6
timeout 400 python bench.py --cache /tmp/c3b.phast > gpurun_out/r9_lbfs.json 2> gpurun_out/r9_lbfs.err; cat gpurun_out/r9_lbfs.json; tail -3 gpurun_out/r9_lbfs.err
PHAST_SWEEP=pipe timeout 400 python bench.py --layout wavefront --cache /tmp/c3w.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r9_pipe.json 2> gpurun_out/r9_pipe.err; cat gpurun_out/r9_pipe.json; tail -3 gpurun_out/r9_pipe.err
for k in 16 32; do PHAST_SWEEP=pipe timeout 300 python bench.py --layout wavefront --k $k --cache /tmp/c3w.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r9_pipe_k$k.json 2>/dev/null; cat gpurun_out/r9_pipe_k$k.json; done
PHAST_SWEEP=pipe timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_pipe -s 3 -c 1 -o /tmp/r9_prof python bench.py --layout wavefront --cache /tmp/c3w.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ncu -i /tmp/r9_prof.ncu-rep --page raw --csv > gpurun_out/r9_prof_raw.csv
ncu -i /tmp/r9_prof.ncu-rep --page details --csv > gpurun_out/r9_prof_details.csv
cp /tmp/r9_prof.ncu-rep gpurun_out/
timeout 300 python bench_diameter.py > gpurun_out/r9_diam.json 2> gpurun_out/r9_diam.err; cat gpurun_out/r9_diam.json
