# ncu of the GEMM-leg TMA setting (bulk 7 on 148 SMs) and of bulk 7 on 112
set -x
mkdir -p /tmp/ncu_leg
for spec in "bulk 7 148" "bulk 7 112"; do
  set -- $spec
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:mp_swap -s 2 -c 2 \
    -o /tmp/ncu_leg/prof_$1_$2_$3 python bench.py --steps 1 --warmup 1 --micro-batches 1 --e2e-steps 1 \
    --no-cpu-baseline --no-gemm --no-autotune --no-duplex --no-configs --path $1 --variant $2 --max-ctas $3 > gpurun_out/ncu_leg_$1_$2_$3.log 2>&1
  python tools/ncu_summary.py full /tmp/ncu_leg/prof_$1_$2_$3.ncu-rep gpurun_out/ncu_leg_$1_$2_$3.json
  ncu -i /tmp/ncu_leg/prof_$1_$2_$3.ncu-rep --page details > gpurun_out/ncu_leg_$1_$2_$3_details.txt 2>&1
done
