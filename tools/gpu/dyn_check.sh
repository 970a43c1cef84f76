# AUTO split: whole GPU suite, the split A/B (blocked vs auto), default bench
set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_dyn.log 2>&1; echo smoke rc $?
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_dyn.log 2>&1; echo pytest rc $?
tail -3 gpurun_out/pytest_gpu_dyn.log
SPLITS=0,3 timeout 900 python tools/split_ab.py 6 > gpurun_out/split_ab_auto.jsonl 2> gpurun_out/split_ab.err; echo ab rc $?
T0=$(date +%s)
timeout 900 python bench.py > gpurun_out/bench_dyn_full.json 2> gpurun_out/bench_dyn_full.err; echo bench rc $?
echo "bench wall s: $(( $(date +%s) - T0 ))"
