// dryrun.cu -- APT's dry-run and bandwidth trials.
#include "common.cuh"
#include "trainer.h"

namespace apt {
apt_status set_err(apt_ctx* c, apt_status s, const char* fmt, ...);
}

extern "C" apt_status apt_dryrun(apt_trainer* t, int64_t, apt_plan_stats*) {
  return apt::set_err(t ? t->ctx : nullptr, APT_E_UNSUPPORTED, "apt_dryrun: not built yet");
}

extern "C" apt_status apt_profile_links(apt_ctx* c, apt_bw_profile*) {
  return apt::set_err(c, APT_E_UNSUPPORTED, "apt_profile_links: not built yet");
}
