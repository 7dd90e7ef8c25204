#!/bin/bash
# k_lane_pk block size (warps per block) x candidates per lane: C5 sweep (makespan only) and
# the e2e batch (makespan + per-device peak memory)
for cfg in "FASTT_PK_WPB=4" "FASTT_PK_WPB=2" "FASTT_PK_WPB=1" "X=1"; do
  echo "== sweep $cfg"; env $cfg python tools/probe.py C5 1000000,1000000 2>&1 | tail -1 | cut -c1-200
done
for cfg in "FASTT_PK_CPL=1" "FASTT_PK_CPL_PEAK=1,FASTT_PK_WPB=4" "FASTT_PK_CPL_PEAK=1,FASTT_PK_WPB=1" "FASTT_PK_CPL_PEAK=1"; do
  echo "== e2e $cfg"; env $(echo $cfg | tr ',' ' ') python tools/e2e_probe.py 1000000 2>&1 | tail -1 | cut -c1-200
done
