# direct shape 9 with the warp-claim kernel (dynamic split) vs blocked
set -x
timeout 900 python -m pytest tests/test_gpu_bounds.py tests/test_gpu_options.py -m gpu -x -q > gpurun_out/pytest_w9.log 2>&1; echo pytest rc $?
tail -2 gpurun_out/pytest_w9.log
SPLITS=0,2 PATHS=direct VARIANTS=9 CASES=0,1,4 CAPS=32,64,96,148 timeout 900 python tools/split_ab.py 4 > gpurun_out/warp9.jsonl 2> gpurun_out/warp9.err; echo ab rc $?
