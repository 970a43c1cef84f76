# capped swap beside a GEMM: paced settings with 20 paired rounds; ncu of the capped shapes
set -x
GEMM_ROUNDS=20 GEMM_COMBOS="direct:7:64;direct:7:64:850000;direct:9:64:850000;direct:11:64:850000;direct:9:96:850000;direct:11:96:850000;direct:11:128:850000;direct:7:148:850000;direct:9:148:850000;direct:11:148:850000;direct:9:64:720000;direct:11:96:720000" timeout 1200 python tools/sweep.py gemm > gpurun_out/capped2_gemm.jsonl 2> gpurun_out/capped2_gemm.err; echo gemm rc $?
mkdir -p /tmp/ncu
for v in 7 9 10 11; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mp_swap -s 2 -c 2 \
    -o /tmp/ncu/prof_capped_v$v python bench.py --steps 1 --warmup 1 --micro-batches 1 --e2e-steps 1 \
    --no-cpu-baseline --no-gemm --no-autotune --no-duplex --no-configs --path direct --variant $v --max-ctas 64 > gpurun_out/ncu_capped_v$v.log 2>&1; echo ncu v$v rc $?
python tools/ncu_summary.py full /tmp/ncu/prof_capped_v$v.ncu-rep gpurun_out/ncu_capped_v$v.json
ncu -i /tmp/ncu/prof_capped_v$v.ncu-rep --page details > gpurun_out/ncu_capped_v${v}_details.txt 2>&1
ncu -i /tmp/ncu/prof_capped_v$v.ncu-rep --page source --csv > /tmp/ncu/src_v$v.csv 2>&1; gzip -c /tmp/ncu/src_v$v.csv > gpurun_out/ncu_capped_v${v}_source.csv.gz
done
ls -la gpurun_out/ /tmp/ncu
