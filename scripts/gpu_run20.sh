set -x
mkdir -p gpurun_out
export PHAST_VERBOSE=1
timeout 600 python -m pytest tests/test_gpu.py -x -q -k "sweep_modes or c1_all or every_k" 2>&1 | tail -3
for R in 65536 32768; do timeout 400 python bench.py --layout diagonal --delta $R --cache /tmp/c3d$R.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r20_d$R.json 2>gpurun_out/r20_d$R.err; cat gpurun_out/r20_d$R.json; tail -2 gpurun_out/r20_d$R.err; done
for R in 65536 32768; do timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r20_launches_d$R.csv python bench.py --layout diagonal --delta $R --cache /tmp/c3d$R.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1; done
