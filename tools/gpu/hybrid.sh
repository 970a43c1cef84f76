# bulk shape 9 (TMA warp + LSU warp, dynamic claims) vs bulk 7 beside the GEMM
set -x
timeout 900 python -m pytest tests/test_gpu_bounds.py tests/test_gpu_variants.py tests/test_gpu_options.py -m gpu -x -q > gpurun_out/pytest_hyb.log 2>&1; echo pytest rc $?
tail -2 gpurun_out/pytest_hyb.log
SPLITS=3 PATHS=bulk VARIANTS=7,9 CASES=0,4 CAPS=148 timeout 600 python tools/split_ab.py 4 > gpurun_out/hyb_alone.jsonl 2> gpurun_out/hyb.err; echo alone rc $?
GEMM_ROUNDS=20 GEMM_COMBOS="bulk:7:148;bulk:9:148;bulk:7:148;bulk:9:148" timeout 900 python tools/sweep.py gemm > gpurun_out/hyb_gemm.jsonl 2>> gpurun_out/hyb.err; echo gemm rc $?
WINDOW=4000 WINDOW_ROUNDS=5 WINDOW_COMBOS="bulk:7:148:0;bulk:9:148:0;direct:9:64:0;bulk:9:148:0" timeout 1200 python tools/sweep.py windows > gpurun_out/hyb_windows.jsonl 2>> gpurun_out/hyb.err; echo windows rc $?
