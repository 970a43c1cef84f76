#!/bin/bash
# Standard measurement set of a round, run on the GPU box (gpurun):
#   bench line, ncu launch list of the same command, one ncu --set full
#   capture of the swap kernels (one swap-out + one swap-in launch), and the
#   same for the capped (GEMM-concurrent) configuration.
# The ncu runs pass --no-autotune: ncu serialises and cache-flushes every
# launch, which distorts mpress_autotune's probe timing, and the probe's own
# kernels would be the first mp_swap launches -s/-c count.  The bench line
# (no ncu) records what autotune chose; --no-autotune runs AUTO's default
# (bulk), which is what it chose on one B200.
# .ncu-rep files stay on the box (/tmp: gpurun copies back <= 64 MiB); their
# summaries (tools/ncu_summary.py, --page details) come back.
# usage: tools/profile_round.sh rNN [extra bench args]
R=${1:-r01}; shift
OUT=gpurun_out/$R
REP=/tmp/ncu_$R
mkdir -p $OUT $REP
python -c "import __graft_entry__ as g; g.build()"
T0=$(date +%s)
timeout 900 python bench.py "$@" > $OUT/bench.json 2> $OUT/bench.err
echo "bench wall s: $(( $(date +%s) - T0 ))" > $OUT/bench_wall.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 3 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-gemm --no-autotune "$@" > $OUT/ncu_launches.log 2>&1
python tools/ncu_summary.py launches $OUT/launches.csv $OUT/launches_summary.json > /dev/null
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mp_swap -s 2 -c 2 \
    -o $REP/prof_swap python bench.py --steps 1 --warmup 1 --micro-batches 1 --e2e-steps 1 \
    --no-cpu-baseline --no-gemm --no-autotune --no-duplex --no-configs "$@" > $OUT/ncu_full.log 2>&1
python tools/ncu_summary.py full $REP/prof_swap.ncu-rep $OUT/ncu_full_swap.json > /dev/null
ncu -i $REP/prof_swap.ncu-rep --page details > $OUT/ncu_full_details.txt 2>&1
cat $OUT/bench.json; tail -3 $OUT/bench.err
# the capped configuration the GEMM leg uses (AUTO, 64 CTAs -> direct shape 9)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mp_swap -s 2 -c 2 \
    -o $REP/prof_swap_capped python bench.py --steps 1 --warmup 1 --micro-batches 1 --e2e-steps 1 \
    --no-cpu-baseline --no-gemm --no-autotune --no-duplex --no-configs --max-ctas 64 "$@" > $OUT/ncu_full_capped.log 2>&1
python tools/ncu_summary.py full $REP/prof_swap_capped.ncu-rep $OUT/ncu_full_swap_capped.json > /dev/null
ncu -i $REP/prof_swap_capped.ncu-rep --page details > $OUT/ncu_full_capped_details.txt 2>&1
