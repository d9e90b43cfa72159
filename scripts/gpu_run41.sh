set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r41_build.log 2>&1 || echo BUILD FAILED
timeout 1500 python -m pytest tests -x -q -m gpu 2>&1 | tail -4
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python bench.py --cache /tmp/c3_r41.phast > gpurun_out/r41_c3.json 2>gpurun_out/r41_c3.err; cat gpurun_out/r41_c3.json
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
for k in 16 32; do timeout 600 $B --cache /tmp/c3_r41.phast --k $k > gpurun_out/r41_c3_k$k.json 2>/dev/null; cat gpurun_out/r41_c3_k$k.json; done
timeout 600 python bench.py --config C1 --k 1 --steps 50 --e2e-steps 20 > gpurun_out/r41_c1.json 2>/dev/null; cat gpurun_out/r41_c1.json
timeout 600 python bench.py --config C2 --k 16 --steps 50 --e2e-steps 10 > gpurun_out/r41_c2.json 2>/dev/null; cat gpurun_out/r41_c2.json
timeout 600 $B --config C2D --k 16 --steps 50 > gpurun_out/r41_c2d.json 2>/dev/null; cat gpurun_out/r41_c2d.json
timeout 900 python bench.py --config C4 --e2e-steps 1 --no-cpu-baseline > gpurun_out/r41_c4.json 2>gpurun_out/r41_c4.err; cat gpurun_out/r41_c4.json
timeout 900 python bench_diameter.py --config C5 > gpurun_out/r41_c5.json 2>gpurun_out/r41_c5.err; cat gpurun_out/r41_c5.json
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r41_launches.csv $B --cache /tmp/c3_r41.phast --steps 1 --warmup 3 > /dev/null 2>&1
timeout 300 ncu --cache-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r41_launches_warm.csv $B --cache /tmp/c3_r41.phast --steps 1 --warmup 3 > /dev/null 2>&1
python tools/launches.py gpurun_out/r41_launches.csv v > gpurun_out/r41_launches.txt 2>&1; head -4 gpurun_out/r41_launches.txt
python tools/launches.py gpurun_out/r41_launches_warm.csv v > gpurun_out/r41_launches_warm.txt 2>&1; head -4 gpurun_out/r41_launches_warm.txt
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k "regex:sweep_kernel<64, 0, 1, 1, 0, 16>" -s 2 -c 1 -o gpurun_out/r41_level0 $B --cache /tmp/c3_r41.phast --steps 1 --warmup 3 > gpurun_out/r41_ncu.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:sweep_top_kernel -s 2 -c 1 -o gpurun_out/r41_top64 $B --cache /tmp/c3_r41.phast --steps 1 --warmup 3 > gpurun_out/r41_ncu_top.log 2>&1
ls gpurun_out/ | grep r41
