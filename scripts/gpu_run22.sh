set -x
mkdir -p gpurun_out
export PHAST_VERBOSE=1
timeout 600 python -m pytest tests/test_gpu.py -x -q -k "sweep_modes and segments" 2>&1 | tail -3
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
timeout 400 $B --cache /tmp/c3b.phast > gpurun_out/r22_lb_launch.json 2>/dev/null; cat gpurun_out/r22_lb_launch.json
for b in 0 1; do PHAST_SEG_BATCH=$b PHAST_SWEEP=segments timeout 400 $B --cache /tmp/c3b.phast > gpurun_out/r22_lb_seg$b.json 2>/dev/null; cat gpurun_out/r22_lb_seg$b.json; done
for b in 0 1; do PHAST_SEG_BATCH=$b PHAST_SEG_CTAS=8 PHAST_SWEEP=segments timeout 400 $B --cache /tmp/c3b.phast > gpurun_out/r22_lb_seg${b}_8.json 2>/dev/null; cat gpurun_out/r22_lb_seg${b}_8.json; done
for b in 0 1; do PHAST_SEG_BATCH=$b PHAST_SEG_CTAS=8 PHAST_SWEEP=segments timeout 400 $B --layout diagonal --delta 65536 --cache /tmp/c3d.phast > gpurun_out/r22_d_seg$b.json 2>/dev/null; cat gpurun_out/r22_d_seg$b.json; done
PHAST_SEG_BATCH=0 PHAST_SEG_CTAS=8 PHAST_SWEEP=segments timeout 600 ncu --set full --import-source on --clock-control none -k regex:sweep_seg -s 3 -c 1 -o gpurun_out/r22_seg_lb python bench.py --cache /tmp/c3b.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
