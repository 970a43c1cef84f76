# GEMM slowdown in the power-capped regime, several swap settings and the copy engines
set -x
WINDOW_ROUNDS=10 WINDOW_COMBOS="direct:9:148:847059;ce:0:0:0;direct:9:148:600000;direct:9:148:400000;direct:7:64:847059;direct:7:64:0;bulk:5:148:847059;ce:0:0:0;direct:9:148:847059" \
  timeout 1500 python tools/sweep.py windows > gpurun_out/windows.jsonl 2> gpurun_out/windows.err; echo rc $?
