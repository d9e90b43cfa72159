set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r31_build.log 2>&1 || echo BUILD FAILED
timeout 1200 python -m pytest tests -x -q -m gpu 2>&1 | tail -5
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 600 python bench.py --cache /tmp/c3.phast > gpurun_out/r31_c3.json 2>gpurun_out/r31_c3.err; cat gpurun_out/r31_c3.json; tail -2 gpurun_out/r31_c3.err
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r31_launches.csv python bench.py --cache /tmp/c3.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
python tools/launches.py gpurun_out/r31_launches.csv > gpurun_out/r31_launches.txt 2>&1; head -40 gpurun_out/r31_launches.txt
