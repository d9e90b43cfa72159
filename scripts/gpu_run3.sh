# round-1 measurement pass: parity, bench (persistent vs per-level), launch list, one full ncu capture
set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -5
python bench.py --cache /tmp/c3.phast > gpurun_out/bench_persist.json 2> gpurun_out/bench_persist.err
cat gpurun_out/bench_persist.json
PHAST_SWEEP=levels python bench.py --cache /tmp/c3.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_levels.json 2>/dev/null
cat gpurun_out/bench_levels.json
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 12 -c 12 --csv --log-file gpurun_out/launches_persist.csv python bench.py --cache /tmp/c3.phast --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_persistent -s 3 -c 1 -o /tmp/prof_persist python bench.py --cache /tmp/c3.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ncu -i /tmp/prof_persist.ncu-rep --page raw --csv > gpurun_out/prof_persist_raw.csv
ncu -i /tmp/prof_persist.ncu-rep --page details --csv > gpurun_out/prof_persist_details.csv
ncu -i /tmp/prof_persist.ncu-rep --page source --csv > gpurun_out/prof_persist_source.csv 2>/dev/null
ls -la /tmp/prof_persist.ncu-rep; cp /tmp/prof_persist.ncu-rep gpurun_out/ 2>/dev/null
du -sh gpurun_out
