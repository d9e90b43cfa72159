set -x
mkdir -p gpurun_out
export PHAST_VERBOSE=1
timeout 600 python -m pytest tests/test_gpu.py -x -q -k "wave" 2>&1 | tail -5
for win in 4 1 16; do PHAST_WAVE_WINDOW=$win PHAST_SWEEP=wave timeout 300 python bench.py --layout wavefront --cache /tmp/c3w.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r19_w$win.json 2>gpurun_out/r19_w$win.err; cat gpurun_out/r19_w$win.json; grep "wave plan\|error\|Error" gpurun_out/r19_w$win.err | head -3; done
PHAST_SWEEP=wave timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none --csv --log-file gpurun_out/r19_launches_wave.csv python bench.py --layout wavefront --cache /tmp/c3w.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
PHAST_SWEEP=wave timeout 600 ncu --set full --import-source on --clock-control none -k regex:sweep_wave -s 3 -c 1 -o gpurun_out/r19_wave python bench.py --layout wavefront --cache /tmp/c3w.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ls -la gpurun_out
