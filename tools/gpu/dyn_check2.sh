# AUTO split with the stride for small launches: split A/B (blocked / strided / auto), capped cases, options + bounds tests
set -x
timeout 900 python -m pytest tests/test_gpu_bounds.py tests/test_gpu_options.py tests/test_gpu_swap.py -m gpu -x -q > gpurun_out/pytest_dyn2.log 2>&1; echo pytest rc $?
tail -2 gpurun_out/pytest_dyn2.log
SPLITS=0,1,3 timeout 900 python tools/split_ab.py 6 > gpurun_out/split_ab_auto2.jsonl 2> gpurun_out/split_ab.err; echo ab rc $?
SPLITS=0,1,3 CAPS=32,64,128 CASES=0,1,2 timeout 900 python tools/split_ab.py 4 >> gpurun_out/split_ab_auto2.jsonl 2>> gpurun_out/split_ab.err; echo ab capped rc $?
