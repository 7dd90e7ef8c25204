#!/bin/bash
# One GPU call's worth of round measurements (run under gpurun from the repo root):
#   1. the bench line (no profiler), 2. the measured int32 pipe peaks
#   (tools/alu_peak.cu, plus its ncu instruction counts), 3. the ncu launch
#   list of a short bench, 4. one `ncu --set full` capture of the main
#   k_sim_lane sweep launch (source page kept), 5. the prep kernels.
# usage: tools/profile_round.sh <tag>
set -u
tag=${1:-r02}
mkdir -p gpurun_out
python bench.py > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gpurun_out/alu_peak tools/alu_peak.cu && \
  ./gpurun_out/alu_peak > gpurun_out/${tag}_alu_peak.json && \
  ncu --metrics smsp__inst_executed.sum,sm__inst_executed_pipe_alu.sum,sm__inst_executed_pipe_fma.sum,sm__cycles_elapsed.avg,gpu__time_duration.sum,sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active \
    --clock-control none -c 5 --csv --log-file gpurun_out/${tag}_alu_peak_ncu.csv ./gpurun_out/alu_peak > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${tag}_launches.csv \
    python bench.py --steps 1 --warmup 3 --candidates 200000 --no-e2e --no-cpu --no-configs > gpurun_out/${tag}_ncu_bench.log 2>&1
# the main sweep launch: the packed-key lane kernel (k_lane_pk) over 300k PIN candidates
ncu --set full --clock-control none --import-source on -k regex:k_lane_pk -c 1 -o gpurun_out/${tag}_k_lane_pk -f \
    python tools/ncu_sim.py 300000 > gpurun_out/${tag}_ncu_full.log 2>&1
ncu -i gpurun_out/${tag}_k_lane_pk.ncu-rep --page raw --csv > gpurun_out/${tag}_k_lane_pk_raw.csv 2>/dev/null
ncu -i gpurun_out/${tag}_k_lane_pk.ncu-rep --page source --csv --print-source sass > gpurun_out/${tag}_k_lane_pk_source.csv 2>/dev/null
# the preparation pipeline's heaviest kernels (split candidates)
ncu --set full --clock-control none --import-source on -k regex:"k_rank|k_sort|k_cards_hdr|k_cards_pred|k_cp" -c 5 -o gpurun_out/${tag}_prep -f \
    python bench.py --steps 1 --warmup 1 --candidates 20000 --no-e2e --no-cpu --no-configs > gpurun_out/${tag}_ncu_prep.log 2>&1
ls -la gpurun_out
