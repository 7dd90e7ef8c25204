// k_sim_lane_inst.cu -- template instances of k_sim_lane for one device-count
// width GSH = FASTT_GSH and one memory mode MM = FASTT_MM (compiled 6 x 3
// times by build.py, -DFASTT_GSH=0..5 -DFASTT_MM=0..2); k_sim_lane.cu
// dispatches through the getters lane_fn_g<GSH>_m<MM>.
#include "k_sim_lane_body.cuh"

#if !defined(FASTT_GSH) || !defined(FASTT_MM)
#error "compile with -DFASTT_GSH=<0..5> -DFASTT_MM=<0..2>"
#endif

namespace fastt {

template <typename T, int CM, bool EX, bool MG, bool PK = false>
static const void *lane_fn_t() {
  return (const void *)k_sim_lane<T, FASTT_GSH, CM, EX, MG, PK, FASTT_MM>;
}
template <bool EX, bool MG> static const void *lane_fn_x(int tbits, int cm, bool pk) {
  if (tbits == 32) {
    if (!MG && pk && cm != 2) return cm == 0 ? lane_fn_t<uint32_t, 0, EX, false, true>() : lane_fn_t<uint32_t, 1, EX, false, true>();
    if (cm == 0) return lane_fn_t<uint32_t, 0, EX, MG>();
    return cm == 1 ? lane_fn_t<uint32_t, 1, EX, MG>() : lane_fn_t<uint32_t, 2, EX, MG>();
  }
  return cm == 2 ? lane_fn_t<uint64_t, 2, EX, MG>() : lane_fn_t<uint64_t, 1, EX, MG>();
}
const void *FASTT_CAT(FASTT_CAT(FASTT_CAT(lane_fn_g, FASTT_GSH), _m), FASTT_MM)(int tbits, int cm, bool exact, bool mg,
                                                                                bool pk) {
  if (mg) return exact ? lane_fn_x<true, true>(tbits, cm, false) : lane_fn_x<false, true>(tbits, cm, false);
  return exact ? lane_fn_x<true, false>(tbits, cm, pk) : lane_fn_x<false, false>(tbits, cm, pk);
}

#if FASTT_MM == 0
// INSERT (R1i) on the lane kernel: base graph, plain keys, no memory mode
template <typename T, int CM, bool EX> static const void *lane_ins_t() {
  return (const void *)k_sim_lane<T, FASTT_GSH, CM, EX, false, false, 0, true>;
}
template <bool EX> static const void *lane_ins_x(int tbits, int cm) {
  if (tbits == 32)
    return cm == 0 ? lane_ins_t<uint32_t, 0, EX>() : cm == 1 ? lane_ins_t<uint32_t, 1, EX>() : lane_ins_t<uint32_t, 2, EX>();
  return cm == 2 ? lane_ins_t<uint64_t, 2, EX>() : lane_ins_t<uint64_t, 1, EX>();
}
const void *FASTT_CAT(lane_ins_fn_g, FASTT_GSH)(int tbits, int cm, bool exact) {
  return exact ? lane_ins_x<true>(tbits, cm) : lane_ins_x<false>(tbits, cm);
}
#endif

}  // namespace fastt
