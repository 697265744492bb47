// strategies.cu -- layer-1 Permute / Shuffle / Execute / Reshuffle of NFP, SNP
// and DNP.  (filled in below)
#include "common.cuh"
#include "trainer.h"

namespace apt {
apt_status set_err(apt_ctx* c, apt_status s, const char* fmt, ...);
apt_status strategy_alloc(apt_trainer* t, RankState&) {
  return set_err(t->ctx, APT_E_UNSUPPORTED, "strategy not built yet");
}
apt_status layer1_fwd_strategy(apt_trainer* t) { return set_err(t->ctx, APT_E_UNSUPPORTED, "strategy not built yet"); }
apt_status layer1_bwd_strategy(apt_trainer* t) { return set_err(t->ctx, APT_E_UNSUPPORTED, "strategy not built yet"); }
}  // namespace apt
