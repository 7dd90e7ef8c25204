// k_sim_inst.cu -- template instances of k_sim for one lane-group width
// GSH = FASTT_GSH (compiled six times by build.py, -DFASTT_GSH=0..5): the
// getter sim_fn_g<GSH> (sim_fn_g0..5) returns the kernel for a (time type, MEM, INS, FC,
// TOPO) combination; k_sim.cu dispatches on GSH.
#include "k_sim_body.cuh"

#ifndef FASTT_GSH
#error "compile with -DFASTT_GSH=<0..5>"
#endif

namespace fastt {

template <typename T, bool FC, bool TOPO>
static const void *sim_fn_m(bool mem, bool ins) {
  constexpr int S = FASTT_GSH;
  if (ins) return mem ? (const void *)k_sim<T, S, true, true, FC, TOPO> : (const void *)k_sim<T, S, false, true, FC, TOPO>;
  return mem ? (const void *)k_sim<T, S, true, false, FC, TOPO> : (const void *)k_sim<T, S, false, false, FC, TOPO>;
}
template <bool TOPO>
static const void *sim_fn_k(int tbits, bool mem, bool ins, bool fc) {
  if (tbits != 32) return sim_fn_m<uint64_t, false, TOPO>(mem, ins);
  return fc ? sim_fn_m<uint32_t, true, TOPO>(mem, ins) : sim_fn_m<uint32_t, false, TOPO>(mem, ins);
}
const void *FASTT_CAT(sim_fn_g, FASTT_GSH)(int tbits, bool mem, bool ins, bool fc, bool topo) {
  return topo ? sim_fn_k<true>(tbits, mem, ins, fc) : sim_fn_k<false>(tbits, mem, ins, fc);
}

}  // namespace fastt
