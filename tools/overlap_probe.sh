#!/bin/bash
# A/B of the C5 1e6 sweep's launch shape (run under gpurun from the repo root):
# candidates per lane x overlap x warp batches of the non-persistent main launch
set -u
for cfg in ${PROBE_CFGS:-"FASTT_PK_CPL=1" "FASTT_PK_CPL=2"}; do
  echo "== $cfg"
  env $(echo $cfg | tr ',' ' ') python tools/probe.py ${PROBE_GRAPHS:-C5} ${PROBE_NS:-1000000,1000000} ${PROBE_FLAGS:-} 2>&1 | tail -2
done
