set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r51_build.log 2>&1 || echo BUILD FAILED
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
for sk in 0 1 2 3; do
PHAST_TOP_SKIP=$sk PHAST_TOP_DEBUG=gpurun_out/r51_top_c1_s$sk.bin timeout 600 $B --config C1 --k 1 --steps 3 --warmup 3 > /dev/null 2>&1
done
timeout 600 ncu --set full --warp-sampling-interval 0 --import-source on --clock-control none -k regex:sweep_top_kernel -s 3 -c 1 -o gpurun_out/r51_top_c1 $B --config C1 --k 1 --steps 1 --warmup 3 > gpurun_out/r51_ncu.log 2>&1; tail -1 gpurun_out/r51_ncu.log
