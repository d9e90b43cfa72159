set -x
mkdir -p gpurun_out
export PHAST_VERBOSE=1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -6
timeout 500 python bench.py --cache /tmp/c3b.phast > gpurun_out/r17.json 2>gpurun_out/r17.err; cat gpurun_out/r17.json; tail -3 gpurun_out/r17.err
for k in 16 32; do timeout 300 python bench.py --k $k --cache /tmp/c3b.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r17_k$k.json 2>/dev/null; cat gpurun_out/r17_k$k.json; done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r17_launches.csv python bench.py --cache /tmp/c3b.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
