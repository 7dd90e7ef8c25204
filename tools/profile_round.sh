#!/bin/bash
# One GPU call's worth of round measurements (run under gpurun from the repo root):
#   1. the bench line (no profiler), 2. the ncu launch list of a short bench,
#   3. one `ncu --set full` capture of the main k_sim_lane sweep launch.
# usage: tools/profile_round.sh <tag>
set -u
tag=${1:-r01f}
mkdir -p gpurun_out
python bench.py > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${tag}_launches.csv \
    python bench.py --steps 1 --warmup 3 --candidates 200000 --no-e2e --no-cpu > gpurun_out/${tag}_ncu_bench.log 2>&1
# the main sweep launch: the lane-per-candidate kernel (k_sim_lane) over 300k PIN candidates
ncu --set full --clock-control none --import-source on -k regex:k_sim_lane -c 1 -o gpurun_out/${tag}_k_sim_lane -f \
    python tools/ncu_sim.py 300000 > gpurun_out/${tag}_ncu_full.log 2>&1
# the preparation pipeline's heaviest kernels (split candidates)
ncu --set full --clock-control none --import-source on -k regex:"k_rank|k_sort|k_cards_hdr|k_cards_pred|k_cp" -c 5 -o gpurun_out/${tag}_prep -f \
    python bench.py --steps 1 --warmup 1 --candidates 20000 --no-e2e --no-cpu > gpurun_out/${tag}_ncu_prep.log 2>&1
ls -la gpurun_out
