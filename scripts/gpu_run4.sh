# wavefront layout + unified persistent kernel: parity, bench A/B, launch list, ncu
set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -5
python bench.py --cache /tmp/c3w.phast > gpurun_out/r4_wave.json 2> gpurun_out/r4_wave.err; cat gpurun_out/r4_wave.json; tail -2 gpurun_out/r4_wave.err
PHAST_SWEEP=persistent python bench.py --cache /tmp/c3w.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r4_wave_nostage.json 2>/dev/null; cat gpurun_out/r4_wave_nostage.json
python bench.py --layout levels --cache /tmp/c3l.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r4_levels.json 2>/dev/null; cat gpurun_out/r4_levels.json
PHAST_SWEEP=levels python bench.py --layout levels --cache /tmp/c3l.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r4_levels_launch.json 2>/dev/null; cat gpurun_out/r4_levels_launch.json
for d in 16384 32768 131072; do python bench.py --delta $d --e2e-steps 0 --no-cpu-baseline --cache /tmp/c3w$d.phast > gpurun_out/r4_delta$d.json 2>/dev/null; cat gpurun_out/r4_delta$d.json; done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none -s 12 -c 12 --csv --log-file gpurun_out/r4_launches.csv python bench.py --cache /tmp/c3w.phast --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_persistent -s 3 -c 1 -o /tmp/r4_prof python bench.py --cache /tmp/c3w.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ncu -i /tmp/r4_prof.ncu-rep --page details --csv > gpurun_out/r4_prof_details.csv
ncu -i /tmp/r4_prof.ncu-rep --page raw --csv > gpurun_out/r4_prof_raw.csv
cp /tmp/r4_prof.ncu-rep gpurun_out/
du -sh gpurun_out
