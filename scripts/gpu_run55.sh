set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r55_build.log 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests -x -q -m gpu -k betweenness 2>&1 | tail -15
timeout 600 python bench_betweenness.py --config C1 --count 1024 --k 64 > gpurun_out/r55_bc_c1.json 2>gpurun_out/r55_bc_c1.err; cat gpurun_out/r55_bc_c1.json; tail -3 gpurun_out/r55_bc_c1.err
timeout 900 python bench_betweenness.py --config C2 --count 64 --k 16 > gpurun_out/r55_bc_c2.json 2>gpurun_out/r55_bc_c2.err; cat gpurun_out/r55_bc_c2.json; tail -3 gpurun_out/r55_bc_c2.err
