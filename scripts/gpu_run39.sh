set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r39_build.log 2>&1 || echo BUILD FAILED
PHAST_TOP_DEBUG=gpurun_out/r39_top_c1.bin timeout 600 python bench.py --e2e-steps 0 --no-cpu-baseline --config C1 --k 1 --steps 3 --warmup 3 > gpurun_out/r39_c1.json 2>&1
PHAST_TOP_DEBUG=gpurun_out/r39_top_c2.bin timeout 600 python bench.py --e2e-steps 0 --no-cpu-baseline --config C2 --k 16 --steps 3 --warmup 3 > gpurun_out/r39_c2.json 2>&1
ls -la gpurun_out/r39*
