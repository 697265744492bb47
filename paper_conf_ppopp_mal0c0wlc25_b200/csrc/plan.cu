// plan.cu -- APT's planner: the Eq. 2 cost model and the
// strategy pick.  The dry-run counters and link trials live in dryrun.cu.
//
// Eq. 2: T = T_build + T_load + T_shuffle + T_train; T_train is the same
// for every strategy and dropped.  T_build is measured by the dry-run
// (P:142); T_load and T_shuffle are volume / bandwidth of the operator that
// moves them, plus a per-call latency alpha (reading Z23: at B200
// speeds a step's exchange is microseconds, where call latency matters).
// Volumes are per rank summed over the dry-run steps; the predicted time of a
// strategy is the slowest rank's (reading Z13).
#include <cmath>

#include "runtime.h"

namespace apt {
apt_status set_err(apt_ctx* c, apt_status s, const char* fmt, ...);
}

extern "C" apt_status apt_select_strategy(const apt_plan_stats* st, const apt_bw_profile* bw, apt_strategy* pick,
                                          double pred_s[4]) {
  using apt::set_err;
  if (!st || !bw || !pick || !pred_s || st->world < 1 || st->world > APT_MAX_RANKS)
    return set_err(nullptr, APT_E_INVALID, "apt_select_strategy: bad arguments");
  for (int o = 0; o < 8; ++o)
    if (!(bw->beta_Bps[o] > 0.0) || bw->alpha_s[o] < 0.0)
      return set_err(nullptr, APT_E_INVALID, "apt_select_strategy: bandwidth profile slot %d invalid", o);
  const double steps = double(st->steps > 0 ? st->steps : 1);
  const double* a = bw->alpha_s;
  const double* b = bw->beta_Bps;
  int best = 0;
  for (int s = 0; s < 4; ++s) {
    double worst = 0.0;
    for (int r = 0; r < st->world; ++r) {
      double t = st->t_build_s[s][r];
      // T_load: feature rows from local HBM and from peer GPUs
      t += double(st->feat_bytes_local[s][r]) / b[APT_OP_LOCAL_GATHER] + steps * a[APT_OP_LOCAL_GATHER];
      if (st->feat_bytes_peer[s][r] > 0)
        t += double(st->feat_bytes_peer[s][r]) / b[APT_OP_PEER_PULL] + steps * a[APT_OP_PEER_PULL];
      if (st->feat_bytes_host[s][r] > 0)   // host tier of the unified store
        t += double(st->feat_bytes_host[s][r]) / b[APT_OP_HOST_GATHER] + steps * a[APT_OP_HOST_GATHER];
      // T_shuffle (+ the graph shuffle, counted in T_build by the paper but
      // modelled here too since the dry-run does not move it over NVLink)
      if (st->n_calls[s][r] > 0) {
        if (s == APT_NFP) {
          t += 2.0 * steps * a[APT_OP_ALLGATHER] + steps * a[APT_OP_REDUCE_SCATTER];
          t += double(st->graph_bytes[s][r]) / b[APT_OP_ALLGATHER];
          t += double(st->hidden_bytes_fwd[s][r]) / b[APT_OP_REDUCE_SCATTER];
          t += double(st->hidden_bytes_bwd[s][r]) / b[APT_OP_ALLGATHER];
          if (st->attn_bytes[s][r] > 0)   // GAT: partial scores and dalpha, two all-reduces per step
            t += 2.0 * steps * a[APT_OP_ALLREDUCE] + double(st->attn_bytes[s][r]) / b[APT_OP_ALLREDUCE];
        } else if (s == APT_SNP || s == APT_DNP) {
          t += 3.0 * steps * a[APT_OP_ALLTOALLV];
          t += double(st->graph_bytes[s][r] + st->hidden_bytes_fwd[s][r] + st->hidden_bytes_bwd[s][r] +
                      st->attn_bytes[s][r]) / b[APT_OP_ALLTOALLV];
        }
      }
      if (st->attn_feat_bytes[s][r] > 0)   // SNP-GAT: destinations' own rows for the scores
        t += double(st->attn_feat_bytes[s][r]) / b[APT_OP_PEER_PULL];
      worst = std::fmax(worst, t);
    }
    pred_s[s] = worst;
    if (worst < pred_s[best]) best = s;
  }
  *pick = apt_strategy(best);
  return APT_OK;
}
