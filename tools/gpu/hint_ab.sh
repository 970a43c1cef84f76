# new tests + evict-first capped shape vs plain, with the bench's GEMM leg (both GEMM shapes)
set -x
timeout 900 python -m pytest tests/test_gpu_options.py tests/test_gpu_variants.py -m gpu -x -q > gpurun_out/pytest_hint.log 2>&1; echo pytest rc $?
tail -3 gpurun_out/pytest_hint.log
for rep in 1 2; do
for spec in "direct:9:148" "direct:12:148" "direct:12:64" "direct:9:64"; do
  timeout 300 python bench.py --steps 20 --warmup 3 --no-configs --no-cpu-baseline --e2e-steps 1 --no-duplex \
      --no-gemm-ce --gemm-swap-candidates "$spec" --no-autotune > /tmp/g.json 2>> gpurun_out/hint_ab.err
  python - "$spec" >> gpurun_out/hint_ab.jsonl <<'PY'
import json, sys
d = json.loads(open("/tmp/g.json").read().strip().splitlines()[-1])
for key in ("gemm_slowdown", "gemm_slowdown_gpt_fc1"):
    g = d[key]
    print(json.dumps({"spec": sys.argv[1], "leg": key, "slowdown": g.get("slowdown"), "ci95": g.get("slowdown_ci95"),
                      "regime": g.get("regime"), "swap_gbs_during": g.get("swap_gbs_during"),
                      "alone_tflops": g.get("alone_tflops"), "alone_cal": d["gemm_cap_calibration"]["alone_gbs_min_over_ranks"]}))
PY
done
done
