set -x
mkdir -p gpurun_out
export PHAST_VERBOSE=1
timeout 600 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -4
timeout 400 python bench.py --cache /tmp/c3b.phast > gpurun_out/r16.json 2>gpurun_out/r16.err; cat gpurun_out/r16.json; tail -2 gpurun_out/r16.err
for k in 16 32; do timeout 300 python bench.py --k $k --cache /tmp/c3b.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r16_k$k.json 2>/dev/null; cat gpurun_out/r16_k$k.json; done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 195 -c 65 --csv --log-file gpurun_out/r16_launches.csv python bench.py --cache /tmp/c3b.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
