set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r63_build.log 2>&1 || echo BUILD FAILED
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 400 --csv --log-file gpurun_out/r63_launches_betweenness_c1.csv python bench_betweenness.py --config C1 --count 64 --k 64 --check 0 > gpurun_out/r63.log 2>&1
tail -2 gpurun_out/r63.log; wc -l gpurun_out/r63_launches_betweenness_c1.csv
