mkdir -p gpurun_out
export PHAST_VERBOSE=1
timeout 600 compute-sanitizer --tool memcheck --show-backtrace device python -m pytest tests/test_gpu.py -k "sweep_modes and pipe-False-0" -x -q 2>&1 | grep -v "^    " | head -60
