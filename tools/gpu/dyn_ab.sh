# MPRESS_SPLIT_DYNAMIC: correctness first (bounds, options, fuzz), then the split A/B
set -x
timeout 900 python -m pytest tests/test_gpu_bounds.py tests/test_gpu_options.py tests/test_gpu_fuzz.py -m gpu -x -q > gpurun_out/pytest_dyn.log 2>&1; echo pytest rc $?
tail -3 gpurun_out/pytest_dyn.log
timeout 900 python tools/split_ab.py 6 > gpurun_out/split_ab.jsonl 2> gpurun_out/split_ab.err; echo ab rc $?
CAPS=64,148 CASES=0 PATHS=bulk,direct timeout 600 python tools/split_ab.py 6 >> gpurun_out/split_ab.jsonl 2>> gpurun_out/split_ab.err; echo ab capped rc $?
for sp in 0 2 0 2; do
  timeout 300 python bench.py --split $sp --no-gemm --no-configs --no-cpu-baseline --e2e-steps 1 --no-duplex >> gpurun_out/bench_dyn.jsonl 2>> gpurun_out/bench_dyn.err; echo bench split $sp rc $?
done
