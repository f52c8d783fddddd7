// Error state, build info and analytic layer sizes of the C ABI.
#include <cstdarg>
#include <cstdio>
#include <cstring>

#include "common.h"

namespace mobius {
static thread_local char g_err[1024] = "";
void set_error(const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
}
}  // namespace mobius

extern "C" const char* mobius_last_error(void) { return mobius::g_err; }

extern "C" const char* mobius_build_info(void) {
  return "libmobius sm_100a: tcgen05/TMEM/TMA GEMM, fused LN/softmax/CE/embedding kernels, "
         "DRAM stage store + HBM ring prefetcher, CUDA-IPC stage-to-stage transport, host AdamW";
}

// mem = xfer = stage weight bytes in the transfer precision (reading #19);
// act_out = [mbs, s, h] activations of the layer output in the path type.
extern "C" int mobius_layer_sizes(const mobius_model_cfg* c, mobius_layer_profile* out, int* n_out) {
  MOBIUS_CHECK_ARG(c && out && n_out, "null argument");
  MOBIUS_CHECK_ARG(c->n_layers >= 1 && c->hidden > 0 && c->n_heads > 0 && c->hidden % c->n_heads == 0 &&
                       c->seq_len > 0 && c->vocab > 0 && c->micro_batch > 0 && c->n_layers + 2 <= MOBIUS_MAX_LAYERS,
                   "bad model config");
  const int64_t h = c->hidden, V = c->vocab, s = c->seq_len;
  const int64_t e = c->dtype == MOBIUS_F32 ? 4 : 2;
  const int64_t act = (int64_t)c->micro_batch * s * h * e;
  const int Lp = c->n_layers + 2;
  for (int i = 0; i < Lp; ++i) {
    int64_t n;
    if (i == 0)
      n = V * h + s * h;
    else if (i == Lp - 1)
      n = 2 * h + h * V;
    else
      n = 12 * h * h + 13 * h;
    mobius_layer_profile& p = out[i];
    std::memset(&p, 0, sizeof(p));
    p.mem_fwd = p.mem_bwd = p.xfer_fwd = p.xfer_bwd = n * e;
    p.act_out = act;
  }
  *n_out = Lp;
  return MOBIUS_OK;
}
