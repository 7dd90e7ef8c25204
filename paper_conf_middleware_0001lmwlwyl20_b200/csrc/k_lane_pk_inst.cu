// k_lane_pk_inst.cu -- template instances of k_lane_pk for one device-count
// width GSH = FASTT_GSH (compiled six times by build.py, -DFASTT_GSH=0..5);
// k_sim_lane.cu dispatches through the getters lane_pk_fn_g<GSH>.
#include "k_lane_pk.cuh"

#ifndef FASTT_GSH
#error "compile with -DFASTT_GSH=<0..5>"
#endif

namespace fastt {

const void *FASTT_CAT(lane_pk_fn_g, FASTT_GSH)(int mm, bool exact) {
  if (exact)
    return mm == 0   ? (const void *)k_lane_pk<FASTT_GSH, true, 0>
           : mm == 1 ? (const void *)k_lane_pk<FASTT_GSH, true, 1>
                     : (const void *)k_lane_pk<FASTT_GSH, true, 2>;
  return mm == 0   ? (const void *)k_lane_pk<FASTT_GSH, false, 0>
         : mm == 1 ? (const void *)k_lane_pk<FASTT_GSH, false, 1>
                   : (const void *)k_lane_pk<FASTT_GSH, false, 2>;
}

}  // namespace fastt
