set -x
mkdir -p gpurun_out
B="python bench.py --e2e-steps 0 --no-cpu-baseline --cache /tmp/c3b.phast"
timeout 400 $B --steps 3 > /dev/null 2>&1
# level-0 launch of the 4th sweep (launch index: 4 batches x 66 + 64) -- capture the biggest sweep_kernel
timeout 900 ncu --set full --import-source on --clock-control none -k regex:sweep_kernel -s 250 -c 12 -o gpurun_out/r27_levels python bench.py --cache /tmp/c3b.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/r27_ncu.log 2>&1
ncu -i gpurun_out/r27_levels.ncu-rep --page raw --csv > gpurun_out/r27_levels_raw.csv 2>/dev/null
ls -la gpurun_out
