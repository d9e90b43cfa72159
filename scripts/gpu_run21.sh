set -x
mkdir -p gpurun_out
export PHAST_VERBOSE=1
timeout 600 python -m pytest tests/test_gpu.py -x -q -k "sweep_modes" 2>&1 | tail -3
for R in 65536 32768; do PHAST_SWEEP=segments timeout 400 python bench.py --layout diagonal --delta $R --cache /tmp/c3d$R.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r21_d$R.json 2>gpurun_out/r21_d$R.err; cat gpurun_out/r21_d$R.json; tail -2 gpurun_out/r21_d$R.err; done
PHAST_SWEEP=segments timeout 400 python bench.py --cache /tmp/c3b.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r21_lb.json 2>gpurun_out/r21_lb.err; cat gpurun_out/r21_lb.json; tail -2 gpurun_out/r21_lb.err
PHAST_SEG_CTAS=8 PHAST_SWEEP=segments timeout 400 python bench.py --layout diagonal --delta 65536 --cache /tmp/c3d65536.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r21_d8.json 2>gpurun_out/r21_d8.err; cat gpurun_out/r21_d8.json
PHAST_SWEEP=segments timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none --csv --log-file gpurun_out/r21_launches_d65536.csv python bench.py --layout diagonal --delta 65536 --cache /tmp/c3d65536.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
