# the bench's own GEMM leg (40 paired rounds, bootstrap CI) for several paced capped settings
set -x
for spec in "direct:7:64" "direct:9:64" "direct:7:148" "direct:9:96" "direct:9:148" "direct:7:96"; do
  for rep in 1 2; do
  timeout 300 python bench.py --steps 20 --warmup 3 --no-configs --no-cpu-baseline --e2e-steps 1 --no-duplex \
      --no-gemm-ce --gemm-swap-candidates "$spec" --no-autotune > /tmp/g.json 2>> gpurun_out/gemm_settings.err
  python - "$spec" >> gpurun_out/gemm_settings.jsonl <<'PY'
import json, sys
d = json.loads(open("/tmp/g.json").read().strip().splitlines()[-1])
g = d["gemm_slowdown"]
print(json.dumps({"spec": sys.argv[1], "slowdown": g.get("slowdown"), "ci95": g.get("slowdown_ci95"),
                  "regime": g.get("regime"), "swap_gbs_during": g.get("swap_gbs_during"),
                  "alone_tflops": g.get("alone_tflops"), "pace": g.get("swap_pace_mbps"),
                  "path": g.get("swap_path"), "clocks": d.get("clocks")}))
PY
  done
done
