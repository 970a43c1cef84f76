# direct kernel with warp-granular claims: tests, then blocked / strided / dynamic / auto
set -x
timeout 900 python -m pytest tests/test_gpu_bounds.py tests/test_gpu_options.py tests/test_gpu_fuzz.py -m gpu -x -q > gpurun_out/pytest_wd.log 2>&1; echo pytest rc $?
tail -2 gpurun_out/pytest_wd.log
SPLITS=0,1,2 PATHS=direct CASES=0,1,2,3,4,6,7 timeout 900 python tools/split_ab.py 4 > gpurun_out/warp_dyn.jsonl 2> gpurun_out/warp_dyn.err; echo ab rc $?
SPLITS=0,2 PATHS=direct CASES=0,1 CAPS=32,64,148 timeout 900 python tools/split_ab.py 4 >> gpurun_out/warp_dyn.jsonl 2>> gpurun_out/warp_dyn.err; echo ab capped rc $?
SPLITS=0,2 PATHS=direct VARIANTS=9 CASES=0 CAPS=64,148 timeout 900 python tools/split_ab.py 4 >> gpurun_out/warp_dyn.jsonl 2>> gpurun_out/warp_dyn.err; echo ab capped9 rc $?
