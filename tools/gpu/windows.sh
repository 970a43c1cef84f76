# GEMM slowdown in the power-capped regime, several swap settings and the copy engines
set -x
WINDOW_ROUNDS=10 WINDOW_COMBOS="ce:0:0:0;direct:9:148:847059;bulk:5:148:847059;bulk:6:148:847059;bulk:5:74:847059;bulk:3:74:847059;direct:9:148:0;bulk:5:148:0;bulk:5:148:600000;direct:12:148:847059;ce:0:0:0;bulk:5:148:847059;direct:9:148:847059" \
  timeout 1500 python tools/sweep.py windows > gpurun_out/windows2.jsonl 2> gpurun_out/windows2.err; echo rc $?
