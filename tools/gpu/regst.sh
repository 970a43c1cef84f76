# bulk shape 9 (TMA loads, register stores) vs shape 7 beside the GEMM
set -x
timeout 900 python -m pytest tests/test_gpu_bounds.py tests/test_gpu_variants.py -m gpu -x -q > gpurun_out/pytest_regst.log 2>&1; echo pytest rc $?
tail -2 gpurun_out/pytest_regst.log
SPLITS=3 PATHS=bulk VARIANTS=7,9 CASES=0 CAPS=64,148 timeout 600 python tools/split_ab.py 4 > gpurun_out/regst_alone.jsonl 2> gpurun_out/regst.err; echo alone rc $?
GEMM_ROUNDS=20 GEMM_COMBOS="bulk:7:148;bulk:9:148;bulk:7:148;bulk:9:148" timeout 900 python tools/sweep.py gemm > gpurun_out/regst_gemm.jsonl 2>> gpurun_out/regst.err; echo gemm rc $?
