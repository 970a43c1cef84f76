# AUTO variant with deep shapes for small launches vs the fixed shapes
set -x
SPLITS=3 PATHS=bulk VARIANTS=-1,3,0 CASES=1,2,6,7 timeout 900 python tools/split_ab.py 4 > gpurun_out/small_shapes3.jsonl 2> gpurun_out/small_shapes.err; echo bulk rc $?
SPLITS=3 PATHS=direct VARIANTS=-1,5,1 CASES=1,2,6,7 timeout 900 python tools/split_ab.py 4 >> gpurun_out/small_shapes3.jsonl 2>> gpurun_out/small_shapes.err; echo direct rc $?
timeout 900 python -m pytest tests/test_gpu_bounds.py tests/test_gpu_swap.py tests/test_gpu_variants.py -m gpu -x -q > gpurun_out/pytest_small.log 2>&1; echo pytest rc $?
tail -2 gpurun_out/pytest_small.log
