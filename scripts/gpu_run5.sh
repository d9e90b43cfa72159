# every command under its own timeout (a hung kernel must never hold the box)
set -x
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -8
timeout 400 python bench.py --cache /tmp/c3w.phast > gpurun_out/r5_wave.json 2> gpurun_out/r5_wave.err; cat gpurun_out/r5_wave.json; tail -3 gpurun_out/r5_wave.err
PHAST_SWEEP=persistent timeout 300 python bench.py --cache /tmp/c3w.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r5_wave_nostage.json 2>/dev/null; cat gpurun_out/r5_wave_nostage.json
timeout 400 python bench.py --layout levels --cache /tmp/c3l.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r5_levels.json 2>/dev/null; cat gpurun_out/r5_levels.json
PHAST_SWEEP=levels timeout 300 python bench.py --layout levels --cache /tmp/c3l.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r5_levels_launch.json 2>/dev/null; cat gpurun_out/r5_levels_launch.json
for k in 16 32; do timeout 300 python bench.py --k $k --cache /tmp/c3w.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r5_k$k.json 2>/dev/null; cat gpurun_out/r5_k$k.json; done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none -s 12 -c 12 --csv --log-file gpurun_out/r5_launches.csv python bench.py --cache /tmp/c3w.phast --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_persistent -s 3 -c 1 -o /tmp/r5_prof python bench.py --cache /tmp/c3w.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ncu -i /tmp/r5_prof.ncu-rep --page details --csv > gpurun_out/r5_prof_details.csv
ncu -i /tmp/r5_prof.ncu-rep --page raw --csv > gpurun_out/r5_prof_raw.csv
cp /tmp/r5_prof.ncu-rep gpurun_out/
timeout 300 python bench_diameter.py > gpurun_out/r5_diam.json 2> gpurun_out/r5_diam.err; cat gpurun_out/r5_diam.json; tail -2 gpurun_out/r5_diam.err
du -sh gpurun_out
