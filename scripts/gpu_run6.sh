set -x
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -8
timeout 400 python bench.py --cache /tmp/c3w.phast > gpurun_out/r6_warp.json 2> gpurun_out/r6_warp.err; cat gpurun_out/r6_warp.json; tail -3 gpurun_out/r6_warp.err
PHAST_SWEEP=staged timeout 300 python bench.py --cache /tmp/c3w.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r6_staged.json 2>/dev/null; cat gpurun_out/r6_staged.json
for k in 16 32; do timeout 300 python bench.py --k $k --cache /tmp/c3w.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r6_k$k.json 2>/dev/null; cat gpurun_out/r6_k$k.json; done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none -s 12 -c 12 --csv --log-file gpurun_out/r6_launches.csv python bench.py --cache /tmp/c3w.phast --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_warp -s 3 -c 1 -o /tmp/r6_prof python bench.py --cache /tmp/c3w.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ncu -i /tmp/r6_prof.ncu-rep --page details --csv > gpurun_out/r6_prof_details.csv
ncu -i /tmp/r6_prof.ncu-rep --page raw --csv > gpurun_out/r6_prof_raw.csv
cp /tmp/r6_prof.ncu-rep gpurun_out/
timeout 300 python bench_diameter.py > gpurun_out/r6_diam.json 2> gpurun_out/r6_diam.err; cat gpurun_out/r6_diam.json
du -sh gpurun_out
