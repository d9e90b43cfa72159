set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r53_build.log 2>&1 || echo BUILD FAILED
timeout 1800 python -m pytest tests -x -q -m gpu --durations=6 2>&1 | tail -10
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/r53_c3.json 2>gpurun_out/r53_c3.err; cat gpurun_out/r53_c3.json
timeout 600 python bench.py --config C1 --k 1 --steps 50 --e2e-steps 20 > gpurun_out/r53_c1.json 2>/dev/null; cat gpurun_out/r53_c1.json
timeout 600 python bench.py --config C2 --k 16 --steps 50 --e2e-steps 10 > gpurun_out/r53_c2.json 2>/dev/null; cat gpurun_out/r53_c2.json
timeout 600 python bench.py --config C2D --k 16 --steps 50 --e2e-steps 0 --no-cpu-baseline > gpurun_out/r53_c2d.json 2>/dev/null; cat gpurun_out/r53_c2d.json
for k in 16 32; do timeout 600 python bench.py --k $k --e2e-steps 0 --no-cpu-baseline > gpurun_out/r53_c3_k$k.json 2>/dev/null; cat gpurun_out/r53_c3_k$k.json; done
