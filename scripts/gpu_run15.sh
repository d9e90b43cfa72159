set -x
mkdir -p gpurun_out
export PHAST_VERBOSE=1
timeout 600 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -4
for t in 65536 262144 16384; do PHAST_TOP_THRESH=$t timeout 300 python bench.py --cache /tmp/c3b.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r15_t$t.json 2>gpurun_out/r15_t$t.err; cat gpurun_out/r15_t$t.json; done
PHAST_TOP_THRESH=0 timeout 300 python bench.py --cache /tmp/c3b.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r15_flat.json 2>/dev/null; cat gpurun_out/r15_flat.json
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 12 -c 30 --csv --log-file gpurun_out/r15_launches.csv python bench.py --cache /tmp/c3b.phast --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
