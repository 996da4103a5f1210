#!/bin/bash
# Round-2 profiling pass (run under gpurun from the repo root).
set -x
mkdir -p gpurun_out
# launch list of the bench command (cold-cache, serialised: compare shares)
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r02.csv \
  python bench.py --steps 2 --warmup 1 --no-extra --no-cpu-baseline --no-e2e > gpurun_out/ncu_bench.log 2>&1
# full capture of the default hot kernel (1M x 192 fp32)
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tsqr_fused -c 1 -o gpurun_out/fused_r02 \
  python tools/run_factor.py --reps 1 > gpurun_out/ncu_fused.log 2>&1
# full capture of the tcgen05 chain kernel (opt-in path)
CAQR_CHAIN=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:tsqr_chain -c 1 \
  -o gpurun_out/chain_tc_r02 python tools/run_factor.py --reps 1 > gpurun_out/ncu_chain.log 2>&1
