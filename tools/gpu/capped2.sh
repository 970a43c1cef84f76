# capped swap beside a GEMM: paced settings with 20 paired rounds; ncu of the capped shapes
set -x
GEMM_ROUNDS=20 GEMM_COMBOS="direct:7:64;direct:7:64:850000;direct:9:64:850000;direct:11:64:850000;direct:9:96:850000;direct:11:96:850000;direct:11:128:850000;direct:7:148:850000;direct:9:148:850000;direct:11:148:850000;direct:9:64:720000;direct:11:96:720000" timeout 1200 python tools/sweep.py gemm > gpurun_out/capped2_gemm.jsonl 2> gpurun_out/capped2_gemm.err; echo gemm rc $?
for v in 7 9 10 11; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mp_swap -s 2 -c 2 \
    -o gpurun_out/prof_capped_v$v python bench.py --steps 1 --warmup 1 --micro-batches 1 --e2e-steps 1 \
    --no-cpu-baseline --no-gemm --no-autotune --no-duplex --no-configs --path direct --variant $v --max-ctas 64 > gpurun_out/ncu_capped_v$v.log 2>&1; echo ncu v$v rc $?
done
