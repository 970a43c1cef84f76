# bulk 9 after the register cap: tests, alone rate, beside the GEMMs
set -x
timeout 900 python -m pytest tests/test_gpu_bounds.py tests/test_gpu_options.py tests/test_gpu_variants.py -m gpu -x -q > gpurun_out/pytest_hc.log 2>&1; echo pytest rc $?
tail -1 gpurun_out/pytest_hc.log
SPLITS=3 PATHS=bulk VARIANTS=7,9 CASES=0 CAPS=148 timeout 600 python tools/split_ab.py 4 > gpurun_out/hc_alone.jsonl 2> gpurun_out/hc.err; echo alone rc $?
GEMM_ROUNDS=20 GEMM_COMBOS="bulk:7:148;bulk:9:148;bulk:9:148" timeout 900 python tools/sweep.py gemm > gpurun_out/hc_gemm.jsonl 2>> gpurun_out/hc.err; echo gemm rc $?
WINDOW=4000 WINDOW_ROUNDS=5 WINDOW_COMBOS="bulk:9:148:0" timeout 600 python tools/sweep.py windows > gpurun_out/hc_windows.jsonl 2>> gpurun_out/hc.err; echo windows rc $?
