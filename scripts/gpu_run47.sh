set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r47_build.log 2>&1 || echo BUILD FAILED
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
show() { python -c "import json,sys;d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]);r=d['roofline'];print(sys.argv[1], round(d['value'],1), 'step', round(d['ms_per_step'],4), 'sweep', round(r['sweep_ms'],4), 'frac', round(r['frac'],3))" $1; }
timeout 600 $B --cache /tmp/c3_r47.phast > gpurun_out/r47_c3_p0.json 2>/dev/null; show gpurun_out/r47_c3_p0.json
for mb in 16 32 48 64 96; do
PHAST_L2_PERSIST_MB=$mb timeout 600 $B --cache /tmp/c3_r47.phast > gpurun_out/r47_c3_p$mb.json 2>/dev/null; show gpurun_out/r47_c3_p$mb.json
done
for mb in 0 32 64; do
PHAST_L2_PERSIST_MB=$mb timeout 600 $B --cache /tmp/c3_r47.phast --k 16 > gpurun_out/r47_c3k16_p$mb.json 2>/dev/null; show gpurun_out/r47_c3k16_p$mb.json
done
PHAST_L2_PERSIST_MB=64 timeout 300 ncu --cache-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r47_launches_p64.csv $B --cache /tmp/c3_r47.phast --steps 1 --warmup 3 > /dev/null 2>&1
python tools/launches.py gpurun_out/r47_launches_p64.csv v > gpurun_out/r47_launches_p64.txt 2>&1; head -3 gpurun_out/r47_launches_p64.txt
