set -x
mkdir -p gpurun_out
export PHAST_VERBOSE=1
timeout 400 python bench.py --cache /tmp/c3b.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r18_levels.json 2>gpurun_out/r18_levels.err; cat gpurun_out/r18_levels.json
for m in wpipe warp pipe staged persistent; do PHAST_SWEEP=$m timeout 300 python bench.py --layout wavefront --cache /tmp/c3w.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r18_$m.json 2>gpurun_out/r18_$m.err; cat gpurun_out/r18_$m.json; tail -2 gpurun_out/r18_$m.err; done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r18_launches_levels.csv python bench.py --cache /tmp/c3b.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
PHAST_SWEEP=wpipe timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none --csv --log-file gpurun_out/r18_launches_wpipe.csv python bench.py --layout wavefront --cache /tmp/c3w.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
