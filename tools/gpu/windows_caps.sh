# bulk 7 at fewer SMs beside the power-capped GEMM
set -x
WINDOW_ROUNDS=10 WINDOW_COMBOS="bulk:7:148:0;bulk:7:128:0;bulk:7:112:0;bulk:7:96:0;bulk:7:74:0;bulk:7:148:0;bulk:7:112:0" timeout 1200 python tools/sweep.py windows > gpurun_out/windows_caps.jsonl 2>&1; echo rc $?
