set -x
mkdir -p gpurun_out
(cd paper_conf_ipps_dellinggnw11_b200/csrc && make -B -j16 > /dev/null 2>&1) || echo BUILD FAILED
timeout 500 python bench.py --cache /tmp/c3b.phast > gpurun_out/r29_c3.json 2>gpurun_out/r29_c3.err; cat gpurun_out/r29_c3.json
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r29_launches.csv python bench.py --cache /tmp/c3b.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:sweep_kernel -s 246 -c 2 -o gpurun_out/r29_levels python bench.py --cache /tmp/c3b.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/r29_ncu.log 2>&1
timeout 900 python bench.py --config C4 --e2e-steps 1 --no-cpu-baseline > gpurun_out/r29_c4.json 2>gpurun_out/r29_c4.err; cat gpurun_out/r29_c4.json; tail -2 gpurun_out/r29_c4.err
timeout 900 python bench_diameter.py --config C5 > gpurun_out/r29_c5.json 2>gpurun_out/r29_c5.err; cat gpurun_out/r29_c5.json; tail -2 gpurun_out/r29_c5.err
