# NEXT-2 replay: the exporter stage with the swap on the direct kernel, the TMA kernel and the copy engines
set -x
timeout 1200 python tools/replay_1f1b.py --stages 8 4 2 --max-ctas 148 --path auto:-1 bulk:7 ce:0 > gpurun_out/replay_paths.jsonl 2> gpurun_out/replay_paths.err; echo rc $?
