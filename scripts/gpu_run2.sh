set -x
nproc
python bench.py --cache /tmp/c3.phast > gpurun_out/bench1.json 2> gpurun_out/bench1.err
tail -3 gpurun_out/bench1.err; cat gpurun_out/bench1.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 195 -c 130 --csv --log-file gpurun_out/launches1.csv python bench.py --cache /tmp/c3.phast --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 186 -c 62 -o gpurun_out/prof1 python bench.py --cache /tmp/c3.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/prof1.log 2>&1
tail -3 gpurun_out/prof1.log
timeout 600 python -m pytest tests -m slow -x -q 2>&1 | tail -5
