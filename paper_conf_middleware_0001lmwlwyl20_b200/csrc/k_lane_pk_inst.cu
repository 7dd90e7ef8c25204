// k_lane_pk_inst.cu -- template instances of k_lane_pk for one device-count
// width GSH = FASTT_GSH (compiled six times by build.py, -DFASTT_GSH=0..5);
// k_sim_lane.cu dispatches through the getters lane_pk_fn_g<GSH>.
#include "k_lane_pk.cuh"

#ifndef FASTT_GSH
#error "compile with -DFASTT_GSH=<0..5>"
#endif

namespace fastt {

const void *FASTT_CAT(lane_pk_fn_g, FASTT_GSH)(int mm, bool exact, int cpl) {
  if (cpl == 4 && mm == 0)  // (four candidates per lane: makespan only)
    return exact ? (const void *)k_lane_pk<FASTT_GSH, true, 0, 4> : (const void *)k_lane_pk<FASTT_GSH, false, 0, 4>;
  if (cpl >= 2 && mm <= 1)  // (two candidates per lane: makespan, + per-device peak memory)
    return exact ? (mm == 0 ? (const void *)k_lane_pk<FASTT_GSH, true, 0, 2> : (const void *)k_lane_pk<FASTT_GSH, true, 1, 2>)
                 : (mm == 0 ? (const void *)k_lane_pk<FASTT_GSH, false, 0, 2>
                            : (const void *)k_lane_pk<FASTT_GSH, false, 1, 2>);
  if (exact)
    return mm == 0   ? (const void *)k_lane_pk<FASTT_GSH, true, 0, 1>
           : mm == 1 ? (const void *)k_lane_pk<FASTT_GSH, true, 1, 1>
                     : (const void *)k_lane_pk<FASTT_GSH, true, 2, 1>;
  return mm == 0   ? (const void *)k_lane_pk<FASTT_GSH, false, 0, 1>
         : mm == 1 ? (const void *)k_lane_pk<FASTT_GSH, false, 1, 1>
                   : (const void *)k_lane_pk<FASTT_GSH, false, 2, 1>;
}

}  // namespace fastt
