# smoke + whole GPU suite + default bench
set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_c.log 2>&1; echo smoke rc $?
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_c.log 2>&1; echo pytest rc $?
tail -2 gpurun_out/pytest_gpu_c.log
SPLITS=3 PATHS=bulk,direct VARIANTS=-1 timeout 900 python tools/split_ab.py 4 > gpurun_out/auto_final.jsonl 2> gpurun_out/auto_final.err; echo ab rc $?
T0=$(date +%s)
timeout 900 python bench.py > gpurun_out/bench_c.json 2> gpurun_out/bench_c.err; echo bench rc $?
echo "bench wall s: $(( $(date +%s) - T0 ))"
