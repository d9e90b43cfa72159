set -x
mkdir -p gpurun_out
export PHAST_VERBOSE=1
timeout 300 python -m pytest tests/test_gpu.py -k sweep_modes -x -q 2>&1 | tail -6
for k in 64 32 16; do PHAST_SWEEP=wpipe timeout 300 python bench.py --layout wavefront --k $k --cache /tmp/c3w.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r14_wp_k$k.json 2>gpurun_out/r14_wp_k$k.err; cat gpurun_out/r14_wp_k$k.json; tail -2 gpurun_out/r14_wp_k$k.err; done
PHAST_SWEEP=wpipe timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_wpipe -s 3 -c 1 -o /tmp/r14_prof python bench.py --layout wavefront --cache /tmp/c3w.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ncu -i /tmp/r14_prof.ncu-rep --page raw --csv > gpurun_out/r14_prof_raw.csv
cp /tmp/r14_prof.ncu-rep gpurun_out/
