// Mobius per-rank runtime (rows a1-a11 of SURVEY §8(a)).
//
//  * Stage store: this rank's stages live in pinned host DRAM in the
//    transfer precision; fp32 master / m / v in host memory (P:L428-434,
//    P:L150-152).
//  * HBM ring of G bytes (the cap of Eq 4/5) with two-ended placement:
//    residence r sits at the bottom (r even) or the top (r odd) of the ring.
//    Loading residence r+1 starts when residence r starts computing and
//    writes only bytes that do not overlap residence r (the Eq 5/6 prefetch
//    P <= G - S); the remainder waits for residence r's release (Eq 9).
//  * Per-GPU schedule (Fig 4): F_{j,1..M} for my stages
//    ascending, then B_{j,1..M} descending; the last stage stays resident.
//  * Stage-input checkpoints are the activation receive slots;
//    backward recomputes the stage forward from them.
//  * Activations / activation-gradients go straight from the producing
//    kernel's epilogue into the consumer rank's slot (CUDA IPC mapping over
//    NVLink), followed by a system-scope release flag (Eq 8).
//  * After B_{j,M}: fp32 dW -> transfer precision, D2H on a side stream,
//    host AdamW on worker threads, overlapping the remaining
//    backward.  The step returns when every update has landed (synchronous
//    update).
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <climits>
#include <cmath>
#include <condition_variable>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <memory>
#include <mutex>
#include <random>
#include <thread>
#include <vector>

#include "common.h"
#include "elem.h"
#include "host.h"
#include "flash.h"
#include "gemm.h"
#include "ops.h"

namespace mobius {

typedef __nv_bfloat16 bf16;

namespace {

inline int64_t al256(int64_t x) { return (x + 255) & ~int64_t(255); }

int64_t now_ns() {
  return std::chrono::duration_cast<std::chrono::nanoseconds>(std::chrono::steady_clock::now().time_since_epoch())
      .count();
}

struct StageDesc {
  int j = 0;                      // global 0-based stage index
  int first = 0, last = 0;        // profile layers [first, last)
  int64_t n_params = 0;           // elements
  int64_t param_off = 0;          // offset in the oracle flat vector
  std::vector<int64_t> layer_off; // element offset of each layer inside the stage blob
  bool has_embed = false, has_head = false;
  int n_blocks = 0;
  int owner = 0;                  // rank (GPU) running the stage
  int ord = 0;                    // index among the owner's stages (ascending)
};

struct PeerInfo {
  int rank;
  cudaIpcMemHandle_t handle;
  int64_t off_ckpt, off_gslot, off_fflag, off_bflag, slot_bytes;
  int n_local, M;
  int64_t off_pf;  // prefetch-chain region: [ticket counter, load_done[R], tickets[R]] (int32)
};

struct Load {           // one residence of a stage in the ring
  int stage_local;      // index into mine
  int end;              // 0 bottom, 1 top
  int64_t base;         // byte offset in the ring
  int64_t bytes;        // footprint in the ring (weights; + dW / staging / recompute workspace, arena mode bwd)
  int64_t copy;         // bytes copied in (the stage weights)
  bool bwd;             // the residence runs the stage's backward
  int64_t wofs = 0;     // offset of the weights in the footprint: 0 at the bottom end; at the top end
                        // the weights sit last (highest addresses), as far as possible from the bottom
                        // residence, so a top prefetch overlaps the running bottom footprint least
};

// byte layout of a backward residence in MOBIUS_FLAG_ARENA_CAP mode, from
// the ring's end inwards: [weights | gradient staging | fp32 dW | nb
// recompute activation sets | (has_embed + nb) activation buffers] at the
// bottom end, mirrored at the top end.  The weights (prefetched) and the
// gradient staging (read by the D2H offload after the pass) sit farthest from
// the other end, where the next residence's workspace would overlap.
struct BwdFootprint {
  int64_t w, gacc, gst, acts, xs, total;
};
inline BwdFootprint bwd_footprint(int64_t np, int esz, int nb, bool has_embed, int64_t acts_bytes,
                                  int64_t slot_bytes, bool top = false) {
  auto al = [](int64_t x) { return (x + 255) & ~int64_t(255); };
  const int64_t W = al(np * esz), GS = al(np * esz), GA = al(np * 4), AC = nb * acts_bytes,
                XS = (nb + (has_embed ? 1 : 0)) * slot_bytes;
  BwdFootprint f;
  f.total = W + GS + GA + AC + XS;
  if (!top) {
    f.w = 0;
    f.gst = W;
    f.gacc = f.gst + GS;
    f.acts = f.gacc + GA;
    f.xs = f.acts + AC;
  } else {
    f.xs = 0;
    f.acts = XS;
    f.gacc = f.acts + AC;
    f.gst = f.gacc + GA;
    f.w = f.gst + GS;
  }
  return f;
}

// The arena behind the ring: offsets of every fixed region (shared by
// mobius_create and mobius_arena_fixed_bytes, so the planner's G_eff and the
// runtime's layout agree by construction).  Arena mode keeps no dW /
// staging here (they live in the backward residences), 5 activation buffers
// (embedding output, forward pingpong, backward pingpong) and one forward
// activation set; with checkpoint offload the checkpoint and gradient slots
// are two banks of M.
struct FixedLayout {
  int64_t gacc, gstage, ckpt, gslot, fflag, bflag, pf, xs, scr, tok, loss, bad, acts, end;
  int xs_slots, slot_sets;
};
inline FixedLayout fixed_layout(const Shape& sh, int esz, bool flash, int M, int n, int max_blocks,
                                int64_t max_params, bool arena, bool offload, int64_t slot, int64_t ring) {
  auto al = [](int64_t x) { return (x + 255) & ~int64_t(255); };
  FixedLayout f;
  int64_t off = al(ring);
  auto take = [&](int64_t bytes) {
    int64_t o = off;
    off += al(bytes);
    return o;
  };
  f.slot_sets = offload ? 2 : n;
  f.xs_slots = arena ? 5 : max_blocks + 3;
  f.gacc = take(arena ? 0 : max_params * 4);
  f.gstage = take(arena ? 0 : max_params * esz);
  f.ckpt = take((int64_t)f.slot_sets * M * slot);
  f.gslot = take((int64_t)f.slot_sets * M * slot);
  f.fflag = take((int64_t)n * M * 4);
  f.bflag = take((int64_t)n * M * 4);
  f.pf = take((1 + 2 * (2 * (int64_t)n)) * 4);  // ticket counter, load_done[R], tickets[R]; R = 2n - 1 loads
  f.xs = take(slot * f.xs_slots);
  f.scr = take(scratch_bytes(sh, esz, true, flash));
  f.tok = take((int64_t)M * sh.mbs * (sh.s + 1) * 4);
  f.loss = take(8);
  f.bad = take(4);
  f.acts = off;  // recompute workspace last (non-arena: its size depends on the keep plan)
  f.end = arena ? f.acts + al(block_acts_bytes(sh, esz, flash)) : f.acts;
  return f;
}

// LM head row chunk in arena mode: MOBIUS_HEAD_ROWS (default 1024) rounded
// down to whole sequences
inline int arena_head_rows(const Shape& sh) {
  int r = 1024;
  if (const char* e = getenv("MOBIUS_HEAD_ROWS")) r = atoi(e);
  r = std::max(sh.s, r / sh.s * sh.s);
  return std::min(r, sh.T());
}

struct EventTimer : KernelTimer {
  struct Rec {
    cudaEvent_t a, b;
    int cls;
    int64_t flops;
  };
  std::vector<Rec> recs;
  std::vector<cudaEvent_t> pool;
  size_t used = 0;
  // Sampling: only every stride-th launch of a class is bracketed by events
  // (stride coprime with the 4 / 8 GEMMs of a block forward / backward, so
  // every GEMM shape is sampled equally); two event records per launch of
  // ~60k launches per step cost ~8% of the step on the host launch path.
  int stride = 7;
  int64_t count[3] = {0, 0, 0};
  std::vector<char> active;
  cudaEvent_t get() {
    if (used == pool.size()) {
      cudaEvent_t e;
      cudaEventCreate(&e);
      pool.push_back(e);
    }
    return pool[used++];
  }
  void begin(int cls, cudaStream_t st) override {
    const bool on = (count[cls]++ % stride) == 0;
    active.push_back(on);
    if (!on) return;
    Rec r;
    r.a = get();
    r.b = nullptr;
    r.cls = cls;
    r.flops = 0;
    cudaEventRecord(r.a, st);
    recs.push_back(r);
  }
  void end(int cls, cudaStream_t st, int64_t flops) override {
    const bool on = active.back();
    active.pop_back();
    if (!on) return;
    Rec& r = recs.back();
    r.b = get();
    r.flops = flops;
    cudaEventRecord(r.b, st);
  }
  void reset() {
    recs.clear();
    used = 0;
    active.clear();
    count[0] = count[1] = count[2] = 0;
  }
  ~EventTimer() {
    for (auto e : pool) cudaEventDestroy(e);
  }
};

}  // namespace

}  // namespace mobius

using namespace mobius;

struct mobius_ctx {
  mobius_model_cfg cfg;
  mobius_plan_t plan;
  mobius_dist dist;
  Shape sh;
  int esz = 2;
  bool poisoned = false;
  int64_t step_count = 0;

  std::vector<StageDesc> all;   // every stage of the plan
  std::vector<int> mine;        // global indices of my stages (ascending)
  std::vector<int> rank_of;     // stage -> rank
  std::vector<Load> loads;      // residences in load order
  std::vector<int> res_f, res_b;  // local stage -> residence index (fwd / bwd)

  // host
  std::vector<void*> h_weights;   // pinned, per local stage, transfer precision
  std::vector<void*> h_grads;     // pinned, per local stage
  std::vector<float*> h_master, h_m, h_v;
  int32_t* h_tokens = nullptr;    // pinned staging of the step's tokens
  int64_t h_tokens_cap = 0;
  double* h_loss = nullptr;
  std::unique_ptr<ThreadPool> pool;

  // device
  uint8_t* arena = nullptr;
  int64_t arena_bytes = 0, ring_bytes = 0;
  uint8_t* ring = nullptr;
  float* grad_acc = nullptr;      // fp32, max local stage params
  uint8_t* grad_stage = nullptr;  // transfer precision, max local stage params
  uint8_t* ckpt = nullptr;        // [n_local][M] act slots (stage inputs)
  uint8_t* gslot = nullptr;       // [n_local][M] act-grad slots
  int* fflag = nullptr;           // [n_local][M]
  int* bflag = nullptr;           // [n_local][M]
  int64_t slot_bytes = 0;
  int max_M = 0;
  uint8_t* acts_base = nullptr;   // per-block saved activations (recompute)
  uint8_t* keep_pool = nullptr;   // kept activations (no recompute) for some stages
  int64_t keep_bytes = 0;
  std::vector<int64_t> keep_off;  // per local stage: offset into keep_pool, -1 if not kept
  std::vector<int> keep_nb;       // per local stage: kept blocks (its LAST keep_nb blocks; the rest recomputed)
  int64_t acts_bytes = 0;
  int64_t keep_acts_bytes = 0;  // per kept block-microbatch (compact layout on the bf16 flash path)
  bool keep_compact = false;
  int max_blocks = 0;
  int ws_blocks = 0;              // recompute workspace entries (acts_base)
  uint8_t* xs_base = nullptr;     // [max_blocks+1] x buffers [T,h]
  uint8_t* scratch_base = nullptr;
  uint8_t* tok_dev = nullptr;
  double* loss_dev = nullptr;
  int64_t off_ckpt = 0, off_gslot = 0, off_fflag = 0, off_bflag = 0, off_pf = 0;
  // cross-GPU prefetch priority chain (mobius_set_prefetch_groups)
  std::vector<int> pf_group;      // uplink group per rank (empty: no chain)
  std::vector<int> pf_pred_rank;  // per my load: rank of its predecessor in the group chain (-1: none / mine)
  std::vector<int> pf_pred_load;  // ... and that rank's load index
  int pf_leader = -1;             // rank holding the group's ticket counter
  int* pf_base = nullptr;         // my prefetch-chain region (arena)
  // MOBIUS_FLAG_DEVICE_TAIL_UPDATE: optimizer state of local stage 0 in HBM
  bool dev_tail = false;
  bool tail_resident = false;     // d_wstage holds local stage 0's current weights (after the first update)
  float* d_opt = nullptr;         // master | m | v, each al256(np0 * 4) bytes
  int64_t d_opt_stride = 0;       // floats between the three
  uint8_t* d_wstage = nullptr;    // new stage-0 weights (transfer precision) for the D2H

  // peers
  std::vector<char> p2p_copy;       // per rank: activations to it go through a local slot + copy engine
  uint8_t* send_stage = nullptr;    // 2 local slots (microbatch parity) staging those sends
  cudaStream_t s_p2p = nullptr;
  cudaEvent_t ev_send[2] = {nullptr, nullptr}, ev_sprod = nullptr;
  std::vector<uint8_t*> peer_base;  // opened IPC bases (nullptr for me)
  std::vector<PeerInfo> peers;
  bool connected = false;

  // streams / events
  cudaStream_t s_comp = nullptr, s_h2d = nullptr, s_d2h = nullptr;
  std::vector<cudaEvent_t> ev_release, ev_loaded;
  std::vector<cudaEvent_t> ev_part_a, ev_part_b;   // per-copy timing (2 parts per load)
  std::vector<int64_t> part_bytes;
  std::vector<cudaEvent_t> ev_gready, ev_d2h;      // per local stage
  cudaEvent_t ev_step0 = nullptr, ev_step1 = nullptr;
  std::vector<cudaEvent_t> ev_wait_a, ev_wait_b;   // exposed load waits
  // timeline (mobius_read_timeline): compute passes and offloads of the last step
  std::vector<cudaEvent_t> ev_pass_a, ev_pass_b;   // per exec entry (2 per local stage)
  std::vector<cudaEvent_t> ev_off_a, ev_off_b;     // per local stage
  std::vector<int> part_stage;                     // global stage of each copy part
  std::vector<char> part_d2d;                      // part served from HBM (device tail update)
  int n_parts_last = 0;

  // update worker
  std::thread upd_thread;
  std::mutex upd_mu;
  std::condition_variable upd_cv, upd_done_cv;
  std::deque<std::pair<int, int64_t>> upd_queue;  // (local stage, AdamW step number)
  int upd_pending = 0;
  std::vector<int64_t> upd_done;  // per local stage: AdamW step of its last finished host update
  int64_t upd_wait_ns = 0;        // host time the issue path spent waiting for updates this step
  bool sync_update = false;       // MOBIUS_SYNC_UPDATE at create: wait for every update inside the step
  bool upd_stop = false;
  int64_t upd_ns = 0;
  int64_t last_bwd_host_ns = 0, last_update_end_ns = 0;

  // stats / trace
  std::vector<int32_t> trace;
  EventTimer timer;
  mobius_step_stats stats;
  int64_t launches_step = 0;
  int* h_bad_tok = nullptr;       // pinned: out-of-range token count (mobius_step_device check)
  // MOBIUS_FLAG_ARENA_CAP / MOBIUS_FLAG_CKPT_OFFLOAD
  bool arena_mode = false, offload = false;
  int xs_fixed = 0;               // fixed activation buffers (pingpong of backward at xs_fixed-2, -1)
  std::vector<void*> h_ckpt;      // pinned, per local stage: its M offloaded checkpoints (nullptr if resident)
  std::vector<char> ck_off;       // per local stage: checkpoint offloaded in forward / uploaded in backward
  std::vector<cudaEvent_t> ev_ckoff;              // [2][M]: last offload of bank slot done (s_d2h)
  std::vector<cudaEvent_t> ev_ckprod;             // [M]: a stage input produced (s_comp)
  std::vector<cudaEvent_t> ev_ckup;               // per local stage: its upload done (s_ckup)
  std::vector<cudaEvent_t> ev_ck_a, ev_ck_b;      // per local stage x {offload, upload}: timeline
  std::vector<cudaEvent_t> ev_ckw_a, ev_ckw_b;    // per local stage: compute waiting on its upload
  cudaEvent_t ev_fwd_off = nullptr;               // all forward offloads issued so far done (s_d2h)
  cudaStream_t s_ckup = nullptr;
  int* bad_tok_dev = nullptr;     // its device counter (arena)

  // Releases everything owned so far: mobius_destroy, and any early return
  // of mobius_create (partially built context held by a unique_ptr).
  ~mobius_ctx() { teardown(); }
  void teardown();
};

void mobius_ctx::teardown() {
  cudaSetDevice(dist.device);
  {
    std::lock_guard<std::mutex> g(upd_mu);
    upd_stop = true;
  }
  upd_cv.notify_all();
  if (upd_thread.joinable()) upd_thread.join();
  if (s_comp) cudaStreamSynchronize(s_comp);
  if (s_h2d) cudaStreamSynchronize(s_h2d);
  if (s_d2h) cudaStreamSynchronize(s_d2h);
  for (auto p : peer_base)
    if (p) cudaIpcCloseMemHandle(p);
  peer_base.clear();
  if (s_ckup) cudaStreamSynchronize(s_ckup);
  if (s_p2p) cudaStreamSynchronize(s_p2p);
  for (cudaEvent_t* e : {&ev_send[0], &ev_send[1], &ev_sprod})
    if (*e) {
      cudaEventDestroy(*e);
      *e = nullptr;
    }
  if (send_stage) cudaFree(send_stage);
  send_stage = nullptr;
  for (auto* v : {&ev_release, &ev_loaded, &ev_part_a, &ev_part_b, &ev_gready, &ev_d2h, &ev_wait_a, &ev_wait_b,
                  &ev_pass_a, &ev_pass_b, &ev_off_a, &ev_off_b, &ev_ckoff, &ev_ckprod, &ev_ckup, &ev_ck_a,
                  &ev_ck_b, &ev_ckw_a, &ev_ckw_b}) {
    for (auto e : *v)
      if (e) cudaEventDestroy(e);
    v->clear();
  }
  if (ev_step0) cudaEventDestroy(ev_step0);
  if (ev_step1) cudaEventDestroy(ev_step1);
  if (ev_fwd_off) cudaEventDestroy(ev_fwd_off);
  ev_step0 = ev_step1 = ev_fwd_off = nullptr;
  for (auto p : h_ckpt)
    if (p) cudaFreeHost(p);
  h_ckpt.clear();
  for (auto p : h_weights)
    if (p) cudaFreeHost(p);
  for (auto p : h_grads)
    if (p) cudaFreeHost(p);
  for (auto p : h_master) std::free(p);
  for (auto p : h_m) std::free(p);
  for (auto p : h_v) std::free(p);
  h_weights.clear();
  h_grads.clear();
  h_master.clear();
  h_m.clear();
  h_v.clear();
  if (h_loss) cudaFreeHost(h_loss);
  if (h_tokens) cudaFreeHost(h_tokens);
  if (h_bad_tok) cudaFreeHost(h_bad_tok);
  h_loss = nullptr;
  h_tokens = nullptr;
  h_bad_tok = nullptr;
  if (arena) cudaFree(arena);
  if (keep_pool) cudaFree(keep_pool);
  if (d_opt) cudaFree(d_opt);
  if (d_wstage) cudaFree(d_wstage);
  arena = keep_pool = d_wstage = nullptr;
  d_opt = nullptr;
  if (s_comp) {
    gemm_release_stream(s_comp);
    cudaStreamDestroy(s_comp);
  }
  if (s_h2d) cudaStreamDestroy(s_h2d);
  if (s_d2h) cudaStreamDestroy(s_d2h);
  if (s_ckup) cudaStreamDestroy(s_ckup);
  if (s_p2p) cudaStreamDestroy(s_p2p);
  s_comp = s_h2d = s_d2h = s_ckup = s_p2p = nullptr;
  cudaGetLastError();  // a failed create must not leave a stale error for the caller's next CUDA call
}

namespace {

#define CU(x)                                                                               \
  do {                                                                                      \
    cudaError_t _e = (x);                                                                   \
    if (_e != cudaSuccess) {                                                                \
      ctx->poisoned = true;                                                                 \
      MOBIUS_FAIL(MOBIUS_ECUDA, "%s failed: %s (%s:%d)", #x, cudaGetErrorString(_e), __FILE__, __LINE__); \
    }                                                                                       \
  } while (0)

#define RC(x)                       \
  do {                              \
    int _rc = (x);                  \
    if (_rc) {                      \
      ctx->poisoned = true;         \
      return _rc;                   \
    }                               \
  } while (0)

int64_t layer_numel(const mobius_model_cfg& c, int i) {
  const int64_t h = c.hidden, V = c.vocab, s = c.seq_len;
  if (i == 0) return V * h + s * h;
  if (i == c.n_layers + 1) return 2 * h + h * V;
  return 12 * h * h + 13 * h;
}

void update_worker(mobius_ctx* ctx) {
  for (;;) {
    int ls;
    int64_t step;
    {
      std::unique_lock<std::mutex> lk(ctx->upd_mu);
      ctx->upd_cv.wait(lk, [&] { return ctx->upd_stop || !ctx->upd_queue.empty(); });
      if (ctx->upd_stop && ctx->upd_queue.empty()) return;
      ls = ctx->upd_queue.front().first;
      step = ctx->upd_queue.front().second;
      ctx->upd_queue.pop_front();
    }
    cudaEventSynchronize(ctx->ev_d2h[ls]);
    int64_t t0 = now_ns();
    const StageDesc& st = ctx->all[ctx->mine[ls]];
    AdamWArgs a{ctx->cfg.lr, ctx->cfg.beta1, ctx->cfg.beta2, ctx->cfg.eps, ctx->cfg.weight_decay, step};
    const int kind = ctx->cfg.dtype == MOBIUS_F32 ? 1 : 0;
    adamw_update(ctx->h_master[ls], ctx->h_m[ls], ctx->h_v[ls], ctx->h_grads[ls], kind, ctx->h_weights[ls], kind,
                 st.n_params, a, *ctx->pool);
    int64_t t1 = now_ns();
    {
      std::lock_guard<std::mutex> g(ctx->upd_mu);
      ctx->upd_ns += t1 - t0;
      ctx->last_update_end_ns = t1;
      ctx->upd_done[ls] = step;
      --ctx->upd_pending;
    }
    ctx->upd_done_cv.notify_all();
  }
}

// Synchronous update across steps: stage ls's host AdamW of
// step `need` must have finished before its weights are swapped in again or
// its gradient landing buffer is overwritten.  Blocks the issuing thread
// only; the GPU keeps running what was issued before.
void wait_update(mobius_ctx* ctx, int ls, int64_t need) {
  if (need <= 0) return;
  std::unique_lock<std::mutex> lk(ctx->upd_mu);
  if (ctx->upd_done[ls] >= need) return;
  const int64_t t0 = now_ns();
  ctx->upd_done_cv.wait(lk, [&] { return ctx->upd_done[ls] >= need || ctx->upd_stop; });
  ctx->upd_wait_ns += now_ns() - t0;
}

// every queued host update finished (the readers and destroy see them)
void drain_updates(mobius_ctx* ctx) {
  std::unique_lock<std::mutex> lk(ctx->upd_mu);
  ctx->upd_done_cv.wait(lk, [&] { return ctx->upd_pending == 0; });
}

void fill_seeded_serial(float* dst, int64_t n, uint64_t seed, int64_t stream_off, float std_) {
  // counter-based N(0, std^2): splitmix64 -> Box-Muller (deterministic per element index)
  for (int64_t i = 0; i < n; ++i) {
    uint64_t z = seed * 0x9E3779B97F4A7C15ull + (uint64_t)(stream_off + i) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    z ^= z >> 31;
    double u1 = ((z >> 11) + 1) * (1.0 / 9007199254740993.0);
    double u2 = ((z & 0x7FF) + 0.5) / 2048.0;
    dst[i] = (float)(std::sqrt(-2.0 * std::log(u1)) * std::cos(6.283185307179586 * u2) * std_);
  }
}

// the same values from the host thread pool (element-indexed: any split gives
// identical numbers); the 13B-width stages hold billions of parameters
thread_local ThreadPool* g_init_pool = nullptr;
void fill_seeded(float* dst, int64_t n, uint64_t seed, int64_t stream_off, float std_) {
  const int64_t chunk = 1 << 20;
  const int tasks = (int)((n + chunk - 1) / chunk);
  if (!g_init_pool || tasks <= 1) return fill_seeded_serial(dst, n, seed, stream_off, std_);
  g_init_pool->parallel_for(tasks, [&](int t) {
    const int64_t b = (int64_t)t * chunk, e = std::min(n, b + chunk);
    fill_seeded_serial(dst + b, e - b, seed, stream_off + b, std_);
  });
}

// initialise the fp32 master of one local stage (oracle init recipe O-1 when
// init_params is NULL: N(0,0.02) weights, N(0,0.02/sqrt(2L)) for w_o/w_2,
// zero biases, unit LN gains)
void seeded_stage_init(const mobius_model_cfg& c, const StageDesc& st, float* out, uint64_t seed) {
  const int64_t h = c.hidden;
  const float proj = 0.02f / std::sqrt(2.0f * c.n_layers);
  for (int li = st.first; li < st.last; ++li) {
    float* p = out + st.layer_off[li - st.first];
    int64_t base = st.param_off + st.layer_off[li - st.first];
    if (li == 0) {
      fill_seeded(p, layer_numel(c, 0), seed, base, 0.02f);
    } else if (li == c.n_layers + 1) {
      for (int64_t i = 0; i < h; ++i) p[i] = 1.f, p[h + i] = 0.f;
      fill_seeded(p + 2 * h, h * (int64_t)c.vocab, seed, base + 2 * h, 0.02f);
    } else {
      BlockLayout L(h);
      for (int64_t i = 0; i < h; ++i) {
        p[L.ln1_g + i] = 1.f;
        p[L.ln1_b + i] = 0.f;
        p[L.ln2_g + i] = 1.f;
        p[L.ln2_b + i] = 0.f;
        p[L.b_o + i] = 0.f;
        p[L.b_2 + i] = 0.f;
      }
      for (int64_t i = 0; i < 3 * h; ++i) p[L.b_qkv + i] = 0.f;
      for (int64_t i = 0; i < 4 * h; ++i) p[L.b_1 + i] = 0.f;
      fill_seeded(p + L.w_qkv, 3 * h * h, seed, base + L.w_qkv, 0.02f);
      fill_seeded(p + L.w_o, h * h, seed, base + L.w_o, proj);
      fill_seeded(p + L.w_1, 4 * h * h, seed, base + L.w_1, 0.02f);
      fill_seeded(p + L.w_2, 4 * h * h, seed, base + L.w_2, proj);
    }
  }
}

template <typename T>
T* tptr(uint8_t* p) {
  return reinterpret_cast<T*>(p);
}

// ---------------------------------------------------------------- step
template <typename T>
struct StepRunner {
  mobius_ctx* ctx;
  const int32_t* tok_dev;
  int M;
  int64_t seq;  // flag value for this step
  float inv_ntok;
  Scratch<T> sc;
  std::vector<BlockActs<T>> acts;
  int64_t h2d_bytes = 0, d2d_bytes = 0;
  int n_parts = 0;

  int64_t ckpt_d2h = 0, ckpt_h2d = 0;
  uint8_t* xrec_base = nullptr;      // backward recompute buffers: xrec(0) embedding output, xrec(b+1) block b output
  std::vector<BlockActs<T>> racts;   // backward recompute activation sets (acts, or the residence's in arena mode)

  T* xbuf(int i) { return tptr<T>(ctx->xs_base + (int64_t)i * ctx->slot_bytes); }
  T* xrec(int i) { return tptr<T>(xrec_base + (int64_t)i * ctx->slot_bytes); }
  // checkpoint / activation-gradient slots: one set of M per local stage, or
  // with checkpoint offload two banks of M (local stage ord uses bank ord % 2)
  int64_t slot_index(int ls, int m) const { return (int64_t)(ctx->offload ? ls % 2 : ls) * M + m; }
  T* ckpt_slot(int ls, int m) { return tptr<T>(ctx->ckpt + slot_index(ls, m) * ctx->slot_bytes); }
  T* grad_slot(int ls, int m) { return tptr<T>(ctx->gslot + slot_index(ls, m) * ctx->slot_bytes); }
  const int32_t* tok(int m) { return tok_dev + (int64_t)m * ctx->sh.mbs * (ctx->sh.s + 1); }

  // destination slot of stage j's output for microbatch m (the input of j+1)
  T* fwd_dest(int j, int m, int** flag) {
    const StageDesc& nx = ctx->all[j + 1];
    int r = nx.owner;
    if (r == ctx->dist.rank) {
      *flag = nullptr;
      return ckpt_slot(nx.ord, m);
    }
    const PeerInfo& pi = ctx->peers[r];
    uint8_t* b = ctx->peer_base[r];
    *flag = reinterpret_cast<int*>(b + pi.off_fflag) + (int64_t)nx.ord * pi.M + m;
    return tptr<T>(b + pi.off_ckpt + ((int64_t)nx.ord * pi.M + m) * pi.slot_bytes);
  }
  // Destination of stage j's forward output for microbatch m.  A peer on
  // another GPU gets it through a local staging slot and a copy-engine
  // transfer over NVLink (send_staged) - the producing GEMM's TMA stores stay
  // local - unless MOBIUS_P2P_DIRECT=1 (the epilogue stores straight into
  // the peer's slot, as it does for a peer sharing this GPU).
  T* fwd_target(int j, int m, int** flag, T** remote) {
    T* d = fwd_dest(j, m, flag);
    *remote = nullptr;
    if (!*flag || !ctx->p2p_copy[ctx->all[j + 1].owner]) return d;
    *remote = d;
    cudaStreamWaitEvent(ctx->s_comp, ctx->ev_send[m % 2], 0);  // the slot's previous send has left
    return tptr<T>(ctx->send_stage + (int64_t)(m % 2) * ctx->slot_bytes);
  }
  int send_staged(const T* local, T* remote, int* flag, int m) {
    CU(cudaEventRecord(ctx->ev_sprod, ctx->s_comp));
    CU(cudaStreamWaitEvent(ctx->s_p2p, ctx->ev_sprod, 0));
    CU(cudaMemcpyAsync(remote, local, (int64_t)ctx->sh.T() * ctx->sh.h * sizeof(T), cudaMemcpyDeviceToDevice,
                       ctx->s_p2p));
    RC(flag_set(flag, (int)seq, ctx->s_p2p));  // after the copy (stream order): release to the consumer
    ++ctx->launches_step;
    CU(cudaEventRecord(ctx->ev_send[m % 2], ctx->s_p2p));
    return MOBIUS_OK;
  }
  // flag after a local producer wrote the output: direct -> set on the compute stream
  int deliver(const T* y, T* remote, int* flag, int m) {
    if (!flag) return MOBIUS_OK;
    if (remote) return send_staged(y, remote, flag, m);
    RC(flag_set(flag, (int)seq, ctx->s_comp));
    ++ctx->launches_step;
    return MOBIUS_OK;
  }

  T* bwd_dest(int j, int m, int** flag) {
    const StageDesc& pv = ctx->all[j - 1];
    int r = pv.owner;
    if (r == ctx->dist.rank) {
      *flag = nullptr;
      return grad_slot(pv.ord, m);
    }
    const PeerInfo& pi = ctx->peers[r];
    uint8_t* b = ctx->peer_base[r];
    *flag = reinterpret_cast<int*>(b + pi.off_bflag) + (int64_t)pv.ord * pi.M + m;
    return tptr<T>(b + pi.off_gslot + ((int64_t)pv.ord * pi.M + m) * pi.slot_bytes);
  }

  // a stage keeps the activations of its last keep_nb blocks (all of them
  // when the budget allows, reading #17); blocks before kf(ls) are recomputed
  bool kept(int ls) const { return ctx->keep_off[ls] >= 0; }
  int kf(int ls) const { return ctx->all[ctx->mine[ls]].n_blocks - ctx->keep_nb[ls]; }
  uint8_t* keep_entry(int ls, int m, int bi) {
    const int64_t e = ctx->keep_acts_bytes + ctx->slot_bytes;
    return ctx->keep_pool + ctx->keep_off[ls] + ((int64_t)m * ctx->keep_nb[ls] + (bi - kf(ls))) * e;
  }
  // input x of block bi of a kept stage (block 0 of an embed stage too)
  T* keep_x(int ls, int m, int bi) { return tptr<T>(keep_entry(ls, m, bi) + ctx->keep_acts_bytes); }
  BlockActs<T> keep_acts(int ls, int m, int bi) {
    BlockActs<T> a;
    carve_block_acts<T>(ctx->sh, keep_entry(ls, m, bi), a, ctx->keep_compact);
    return a;
  }

  const T* stage_w(int res, const StageDesc& st, int layer) {
    return tptr<T>(ctx->ring + ctx->loads[res].base + ctx->loads[res].wofs) + st.layer_off[layer - st.first];
  }

  int issue_part(int r, int64_t b0, int64_t b1) {
    if (b1 <= b0) return MOBIUS_OK;
    const Load& L = ctx->loads[r];
    const StageDesc& st = ctx->all[ctx->mine[L.stage_local]];
    (void)st;
    uint8_t* dst = ctx->ring + L.base + L.wofs + b0;
    // device tail update: local stage 0's weights already live in HBM
    const bool d2d = ctx->tail_resident && L.stage_local == 0;
    if (!d2d) wait_update(ctx, L.stage_local, ctx->step_count);  // the previous step's update of this stage landed
    const uint8_t* src = d2d ? ctx->d_wstage + b0 : (const uint8_t*)ctx->h_weights[L.stage_local] + b0;
    cudaEvent_t a = ctx->ev_part_a[n_parts], b = ctx->ev_part_b[n_parts];
    CU(cudaEventRecord(a, ctx->s_h2d));
    CU(cudaMemcpyAsync(dst, src, b1 - b0, d2d ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, ctx->s_h2d));
    CU(cudaEventRecord(b, ctx->s_h2d));
    ctx->part_bytes[n_parts] = d2d ? 0 : b1 - b0;  // the per-copy GB/s statistics are host-link copies
    ctx->part_stage[n_parts] = ctx->mine[L.stage_local];
    ctx->part_d2d[n_parts] = d2d;
    ++n_parts;
    if (d2d)
      d2d_bytes += b1 - b0;
    else
      h2d_bytes += b1 - b0;
    return MOBIUS_OK;
  }

  // byte split of residence r: [0, split) does not overlap residence r-1 for a
  // bottom load; for a top load the non-overlapping bytes are [split, S)
  void split_of(int r, int64_t& first0, int64_t& first1, int64_t& second0, int64_t& second1) {
    const Load& L = ctx->loads[r];
    const int64_t S = L.copy, G = ctx->ring_bytes;  // the copied bytes vs the previous footprint
    if (r == 0) {
      first0 = 0, first1 = S, second0 = second1 = 0;
      return;
    }
    const Load& P = ctx->loads[r - 1];
    if (L.end == 0) {  // bottom [0,S) vs top [P.base, G)
      int64_t a = std::min(S, P.base);
      first0 = 0, first1 = a, second0 = a, second1 = S;
    } else {           // top copy [L.base + wofs, +S) vs bottom [0, P.bytes)
      int64_t ov = std::max<int64_t>(0, std::min(S, P.bytes - (L.base + L.wofs)));
      first0 = ov, first1 = S, second0 = 0, second1 = ov;
    }
    (void)G;
  }

  // arena mode: a backward residence holds its stage's gradient staging,
  // read by the D2H offload after the release - overwrite only after it
  int wait_offload_of(int r) {
    const Load& P = ctx->loads[r];
    if (ctx->arena_mode && P.bwd) CU(cudaStreamWaitEvent(ctx->s_h2d, ctx->ev_d2h[P.stage_local], 0));
    return MOBIUS_OK;
  }
  // cross-GPU prefetch priority: my load r waits until its predecessor in
  // the uplink group's chain (a load of another rank serving an earlier
  // stage) has landed, then takes a ticket from the group counter
  int* peer_pf(int rank) {
    if (rank == ctx->dist.rank) return ctx->pf_base;
    return reinterpret_cast<int*>(ctx->peer_base[rank] + ctx->peers[rank].off_pf);
  }
  int chain_enter(int r) {
    if (ctx->pf_group.empty()) return MOBIUS_OK;
    const int pr = ctx->pf_pred_rank[r];
    if (pr >= 0) {
      RC(flag_wait(peer_pf(pr) + 1 + ctx->pf_pred_load[r], (int)seq, ctx->s_h2d));
      ++ctx->launches_step;
    }
    const int R = (int)ctx->loads.size();
    RC(ticket_take(peer_pf(ctx->pf_leader), ctx->pf_base + 1 + R + r, ctx->s_h2d));
    ++ctx->launches_step;
    return MOBIUS_OK;
  }
  int chain_leave(int r) {
    if (ctx->pf_group.empty()) return MOBIUS_OK;
    RC(flag_set(ctx->pf_base + 1 + r, (int)seq, ctx->s_h2d));
    ++ctx->launches_step;
    return MOBIUS_OK;
  }

  int load_first_part(int r) {  // issued when residence r-1 starts computing
    if (r >= (int)ctx->loads.size()) return MOBIUS_OK;
    if (r >= 2) {
      CU(cudaStreamWaitEvent(ctx->s_h2d, ctx->ev_release[r - 2], 0));
      RC(wait_offload_of(r - 2));
    }
    RC(chain_enter(r));
    int64_t a0, a1, b0, b1;
    split_of(r, a0, a1, b0, b1);
    return issue_part(r, a0, a1);
  }
  int load_second_part(int r) {  // issued right after residence r-1's release
    if (r >= (int)ctx->loads.size()) return MOBIUS_OK;
    int64_t a0, a1, b0, b1;
    split_of(r, a0, a1, b0, b1);
    if (r >= 1 && b1 > b0) {
      CU(cudaStreamWaitEvent(ctx->s_h2d, ctx->ev_release[r - 1], 0));
      RC(wait_offload_of(r - 1));
    }
    RC(issue_part(r, b0, b1));
    CU(cudaEventRecord(ctx->ev_loaded[r], ctx->s_h2d));
    RC(chain_leave(r));
    return MOBIUS_OK;
  }

  int wait_loaded(int r) {
    CU(cudaEventRecord(ctx->ev_wait_a[r], ctx->s_comp));
    CU(cudaStreamWaitEvent(ctx->s_comp, ctx->ev_loaded[r], 0));
    CU(cudaEventRecord(ctx->ev_wait_b[r], ctx->s_comp));
    return MOBIUS_OK;
  }

  void tr(int op, int j, int m) {
    ctx->trace.push_back(op);
    ctx->trace.push_back(j + 1);
    ctx->trace.push_back(m + 1);
  }

  // ---------------- F_{j,m}
  int forward(int ls, int res, int m) {
    const StageDesc& st = ctx->all[ctx->mine[ls]];
    const Shape& sh = ctx->sh;
    cudaStream_t s = ctx->s_comp;
    tr(0, st.j, m);
    const bool last_stage = st.j == ctx->plan.n_stages - 1;
    const T* x = nullptr;
    if (st.has_embed) {
      T* out;
      int* flag = nullptr;
      T* remote = nullptr;
      if (st.n_blocks == 0 && !last_stage)
        out = fwd_target(st.j, m, &flag, &remote);
      else
        out = (kept(ls) && kf(ls) == 0) ? keep_x(ls, m, 0) : xbuf(0);
      RC(embed_layer_fwd<T>(sh, stage_w(res, st, 0), tok(m), out, s));
      RC(deliver(out, remote, flag, m));
      x = out;
    } else {
      if (ctx->all[st.j - 1].owner != ctx->dist.rank)
        { RC(flag_wait(ctx->fflag + (int64_t)st.ord * M + m, (int)seq, s)); ++ctx->launches_step; }
      x = ckpt_slot(ls, m);
    }
    if (last_stage) return MOBIUS_OK;  // head runs fused with backward (B_{K,m} recomputes it)
    int bi = 0;
    for (int li = st.first; li < st.last; ++li) {
      if (li == 0) continue;
      const bool last_block = (bi == st.n_blocks - 1);
      int* flag = nullptr;
      T* remote = nullptr;
      if (kept(ls) && bi >= kf(ls)) {  // keep this block's activations for its backward (no recompute)
        T* y = last_block ? fwd_target(st.j, m, &flag, &remote) : keep_x(ls, m, bi + 1);
        BlockActs<T> ka = keep_acts(ls, m, bi);
        ka.x = x;
        RC(block_fwd<T>(sh, stage_w(res, st, li), ka, y, sc, s));
        RC(deliver(y, remote, flag, m));
        x = y;
        ++bi;
        continue;
      }
      T* y = last_block ? fwd_target(st.j, m, &flag, &remote)
                        : (kept(ls) && bi + 1 == kf(ls)) ? keep_x(ls, m, bi + 1) : xbuf(1 + (bi % 2));
      acts[0].x = x;
      RC(block_fwd<T>(sh, stage_w(res, st, li), acts[0], y, sc, s));
      RC(deliver(y, remote, flag, m));
      x = y;
      ++bi;
    }
    return MOBIUS_OK;
  }

  // ---------------- B_{j,m}
  int backward(int ls, int res, int m) {
    const StageDesc& st = ctx->all[ctx->mine[ls]];
    const Shape& sh = ctx->sh;
    cudaStream_t s = ctx->s_comp;
    tr(1, st.j, m);
    const T* x;
    int bi = 0;
    std::vector<BlockActs<T>> kacts;
    if (kept(ls)) {  // activations of blocks >= kf kept from F_{j,m}: no recompute for them
      const int k0 = kf(ls);
      for (int b = k0; b < st.n_blocks; ++b) {
        kacts.push_back(keep_acts(ls, m, b));
        kacts.back().x = (b == 0) ? (st.has_embed ? keep_x(ls, m, 0) : ckpt_slot(ls, m)) : keep_x(ls, m, b);
      }
      if (k0 > 0) {  // recompute blocks [0, k0) from the stage input (their outputs match the kept inputs)
        if (st.has_embed) {
          RC(embed_layer_fwd<T>(sh, stage_w(res, st, 0), tok(m), xrec(0), s));
          x = xrec(0);
        } else {
          x = ckpt_slot(ls, m);
        }
        int b = 0;
        for (int li = st.first; li < st.last && b < k0; ++li) {
          if (li == 0 || li == ctx->cfg.n_layers + 1) continue;
          T* y = xrec(b + 1);
          racts[b].x = x;
          RC(block_fwd<T>(sh, stage_w(res, st, li), racts[b], y, sc, s));
          x = y;
          ++b;
        }
      }
      bi = st.n_blocks;
      x = nullptr;  // the head is never in a kept stage
    } else {
      // recompute the stage forward from the checkpoint (a5/a7)
      if (st.has_embed) {
        RC(embed_layer_fwd<T>(sh, stage_w(res, st, 0), tok(m), xrec(0), s));
        x = xrec(0);
      } else {
        x = ckpt_slot(ls, m);
      }
      for (int li = st.first; li < st.last; ++li) {
        if (li == 0 || li == ctx->cfg.n_layers + 1) continue;
        T* y = xrec(bi + 1);
        racts[bi].x = x;
        RC(block_fwd<T>(sh, stage_w(res, st, li), racts[bi], y, sc, s));
        x = y;
        ++bi;
      }
    }
    // gradient w.r.t. the stage output
    const T* dy;
    T* pingpong[2] = {xbuf(ctx->xs_fixed - 2), xbuf(ctx->xs_fixed - 1)};
    int pp = 0;
    if (st.has_head) {
      const int hl = ctx->cfg.n_layers + 1;
      float* G = ctx->grad_acc + st.layer_off[hl - st.first];
      T* dx = pingpong[pp];
      pp ^= 1;
      RC(head_layer_fwd_bwd<T>(sh, stage_w(res, st, hl), x, tok(m), inv_ntok, dx, G, ctx->loss_dev, sc, s));
      dy = dx;
    } else {
      if (ctx->all[st.j + 1].owner != ctx->dist.rank)
        { RC(flag_wait(ctx->bflag + (int64_t)st.ord * M + m, (int)seq, s)); ++ctx->launches_step; }
      dy = grad_slot(ls, m);
    }
    // blocks in reverse
    for (int li = st.last - 1; li >= st.first; --li) {
      if (li == 0 || li == ctx->cfg.n_layers + 1) continue;
      --bi;
      const bool first_block = (bi == 0);
      int* flag = nullptr;
      T* dx;
      if (first_block && !st.has_embed)
        dx = bwd_dest(st.j, m, &flag);
      else {
        dx = pingpong[pp];
        pp ^= 1;
      }
      float* G = ctx->grad_acc + st.layer_off[li - st.first];
      RC(block_bwd<T>(sh, stage_w(res, st, li), (kept(ls) && bi >= kf(ls)) ? kacts[bi - kf(ls)] : racts[bi], dy, dx,
                      G, sc, s));
      if (flag) { RC(flag_set(flag, (int)seq, s)); ++ctx->launches_step; }
      dy = dx;
    }
    if (st.has_embed) {
      RC(embed_layer_bwd<T>(sh, stage_w(res, st, 0), tok(m), dy, ctx->grad_acc, s));
    } else if (st.n_blocks == 0) {
      // head-only stage: pass the head's input gradient upstream
      int* flag = nullptr;
      T* dst = bwd_dest(st.j, m, &flag);
      CU(cudaMemcpyAsync(dst, dy, (int64_t)sh.T() * sh.h * sizeof(T), cudaMemcpyDeviceToDevice, s));
      if (flag) { RC(flag_set(flag, (int)seq, s)); ++ctx->launches_step; }
    }
    return MOBIUS_OK;
  }

  int finish_stage_grads(int ls) {
    const StageDesc& st = ctx->all[ctx->mine[ls]];
    cudaStream_t s = ctx->s_comp;
    // staging buffer reuse: previous offload must have drained
    if (ls + 1 < (int)ctx->mine.size()) CU(cudaStreamWaitEvent(s, ctx->ev_d2h[ls + 1], 0));
    RC(cast_from_f32<T>(ctx->grad_acc, tptr<T>(ctx->grad_stage), st.n_params, s));
    ++ctx->launches_step;
    const bool dev_upd = ctx->dev_tail && ls == 0;
    if (dev_upd) {  // AdamW on the GPU; the new weights go to the pinned store instead of the gradient
      const AdamWArgs a{ctx->cfg.lr, ctx->cfg.beta1, ctx->cfg.beta2, ctx->cfg.eps, ctx->cfg.weight_decay,
                        ctx->step_count + 1};
      const float bc1 = (float)(1.0 - std::pow((double)a.beta1, (double)a.step));
      const float bc2 = (float)(1.0 - std::pow((double)a.beta2, (double)a.step));
      float* w = ctx->d_opt;
      RC(adamw_device<T>(w, w + ctx->d_opt_stride, w + 2 * ctx->d_opt_stride, tptr<T>(ctx->grad_stage),
                         tptr<T>(ctx->d_wstage), st.n_params, a.lr, a.beta1, a.beta2, a.eps, a.wd, bc1, bc2, s));
      ++ctx->launches_step;
    }
    CU(cudaEventRecord(ctx->ev_gready[ls], s));
    CU(cudaStreamWaitEvent(ctx->s_d2h, ctx->ev_gready[ls], 0));
    CU(cudaEventRecord(ctx->ev_off_a[ls], ctx->s_d2h));
    if (!dev_upd) {  // the device-updated stage's weights stay in HBM (d_wstage): nothing crosses the link
      wait_update(ctx, ls, ctx->step_count);  // the previous step's update has read h_grads[ls]
      CU(cudaMemcpyAsync(ctx->h_grads[ls], ctx->grad_stage, st.n_params * sizeof(T), cudaMemcpyDeviceToHost,
                         ctx->s_d2h));
      ctx->stats.d2h_bytes += st.n_params * sizeof(T);
    }
    CU(cudaEventRecord(ctx->ev_off_b[ls], ctx->s_d2h));
    CU(cudaEventRecord(ctx->ev_d2h[ls], ctx->s_d2h));
    if (dev_upd) return MOBIUS_OK;
    {
      std::lock_guard<std::mutex> g(ctx->upd_mu);
      ctx->upd_queue.push_back({ls, ctx->step_count + 1});
      ++ctx->upd_pending;
    }
    ctx->upd_cv.notify_one();
    return MOBIUS_OK;
  }

  // arena mode: this backward residence's workspace may overlap the other
  // end's previous residence, whose gradient staging the D2H offload may
  // still be reading - wait for that offload only when the ranges meet
  int wait_staging_overlap(int res) {
    const Load& L = ctx->loads[res];
    const Load& P = ctx->loads[res - 1];
    const StageDesc& sl = ctx->all[ctx->mine[L.stage_local]];
    const StageDesc& sp = ctx->all[ctx->mine[P.stage_local]];
    const BwdFootprint fl = bwd_footprint(sl.n_params, ctx->esz, sl.n_blocks, sl.has_embed, ctx->acts_bytes,
                                          ctx->slot_bytes, L.end == 1);
    const BwdFootprint fp = bwd_footprint(sp.n_params, ctx->esz, sp.n_blocks, sp.has_embed, ctx->acts_bytes,
                                          ctx->slot_bytes, P.end == 1);
    // workspace of L: its footprint minus the weights
    const int64_t w0 = L.base + (L.end == 1 ? 0 : fl.gst), w1 = L.base + (L.end == 1 ? fl.w : fl.total);
    const int64_t s0 = P.base + fp.gst, s1 = s0 + al256(sp.n_params * ctx->esz);
    if (w0 < s1 && s0 < w1) CU(cudaStreamWaitEvent(ctx->s_comp, ctx->ev_d2h[P.stage_local], 0));
    return MOBIUS_OK;
  }

  // backward buffers of local stage ls in residence res: the fixed
  // workspace, or (arena mode) the residence's own dW / staging / recompute
  // region behind the weights
  void prepare_bwd(int ls, int res) {
    if (!ctx->arena_mode) {
      xrec_base = ctx->xs_base;
      racts = acts;
      return;
    }
    const StageDesc& st = ctx->all[ctx->mine[ls]];
    const BwdFootprint f = bwd_footprint(st.n_params, ctx->esz, st.n_blocks, st.has_embed, ctx->acts_bytes,
                                         ctx->slot_bytes, ctx->loads[res].end == 1);
    uint8_t* base = ctx->ring + ctx->loads[res].base;
    ctx->grad_acc = reinterpret_cast<float*>(base + f.gacc);
    ctx->grad_stage = base + f.gst;
    racts.resize(std::max(1, st.n_blocks));
    for (int b = 0; b < st.n_blocks; ++b) carve_block_acts<T>(ctx->sh, base + f.acts + b * ctx->acts_bytes, racts[b]);
    // xrec(0) is the embedding output (embedding stages only)
    xrec_base = base + f.xs - (st.has_embed ? 0 : ctx->slot_bytes);
  }

  // ---- checkpoint offload (A_Mobius), world size 1
  // stage k's input slot (bank k % 2) is overwritten by stage k+2's input:
  // offloaded right after F_{k-1,m} produced it, uploaded after B_{k+2}
  int ckpt_offload(int k, int m) {
    const int64_t sb = ctx->slot_bytes;
    CU(cudaEventRecord(ctx->ev_ckprod[m], ctx->s_comp));
    CU(cudaStreamWaitEvent(ctx->s_d2h, ctx->ev_ckprod[m], 0));
    if (m == 0) CU(cudaEventRecord(ctx->ev_ck_a[2 * k], ctx->s_d2h));
    CU(cudaMemcpyAsync((uint8_t*)ctx->h_ckpt[k] + m * sb, ckpt_slot(k, m), sb, cudaMemcpyDeviceToHost, ctx->s_d2h));
    CU(cudaEventRecord(ctx->ev_ckoff[slot_index(k, m)], ctx->s_d2h));
    if (m == M - 1) {
      CU(cudaEventRecord(ctx->ev_ck_b[2 * k], ctx->s_d2h));
      CU(cudaEventRecord(ctx->ev_fwd_off, ctx->s_d2h));
    }
    ckpt_d2h += sb;
    return MOBIUS_OK;
  }
  int ckpt_upload(int k, cudaEvent_t after) {
    const int64_t sb = ctx->slot_bytes;
    CU(cudaStreamWaitEvent(ctx->s_ckup, after, 0));
    CU(cudaStreamWaitEvent(ctx->s_ckup, ctx->ev_fwd_off, 0));
    CU(cudaEventRecord(ctx->ev_ck_a[2 * k + 1], ctx->s_ckup));
    for (int m = 0; m < M; ++m)
      CU(cudaMemcpyAsync(ckpt_slot(k, m), (uint8_t*)ctx->h_ckpt[k] + m * sb, sb, cudaMemcpyHostToDevice,
                         ctx->s_ckup));
    CU(cudaEventRecord(ctx->ev_ck_b[2 * k + 1], ctx->s_ckup));
    CU(cudaEventRecord(ctx->ev_ckup[k], ctx->s_ckup));
    ckpt_h2d += M * sb;
    return MOBIUS_OK;
  }

  int run() {
    const int n = (int)ctx->mine.size();
    cudaStream_t s = ctx->s_comp;
    // exec list: F of my stages ascending, then B descending (Fig 4)
    struct Exec {
      int fwd, ls, res;
      bool first_of_res, last_of_res;
    };
    std::vector<Exec> ex;
    for (int k = 0; k < n; ++k) ex.push_back({1, k, ctx->res_f[k], true, k != n - 1});
    for (int k = n - 1; k >= 0; --k) ex.push_back({0, k, ctx->res_b[k], k != n - 1, true});
    RC(load_first_part(0));
    RC(load_second_part(0));
    std::vector<int> bwd_xi(n, -1);
    for (size_t xi = 0; xi < ex.size(); ++xi) {
      const Exec& e = ex[xi];
      if (e.first_of_res) {
        RC(wait_loaded(e.res));
        RC(load_first_part(e.res + 1));  // prefetch of the next residence starts with this one
      }
      CU(cudaEventRecord(ctx->ev_pass_a[xi], s));
      if (!e.fwd) {
        if (ctx->arena_mode && e.res >= 1 && ctx->loads[e.res - 1].bwd) RC(wait_staging_overlap(e.res));
        prepare_bwd(e.ls, e.res);
        if (ctx->ck_off[e.ls]) {  // this stage's checkpoints come back from DRAM
          CU(cudaEventRecord(ctx->ev_ckw_a[e.ls], s));
          CU(cudaStreamWaitEvent(s, ctx->ev_ckup[e.ls], 0));
          CU(cudaEventRecord(ctx->ev_ckw_b[e.ls], s));
        }
        CU(cudaMemsetAsync(ctx->grad_acc, 0, ctx->all[ctx->mine[e.ls]].n_params * 4, s));
      }
      for (int m = 0; m < M; ++m) {
        if (e.fwd) {
          // the output slot (input of stage ls+1) last held stage ls-1's input:
          // its offload must have finished
          if (e.ls + 1 < n && e.ls >= 1 && ctx->ck_off[e.ls - 1])
            CU(cudaStreamWaitEvent(s, ctx->ev_ckoff[slot_index(e.ls + 1, m)], 0));
          RC(forward(e.ls, e.res, m));
          if (e.ls + 1 < n && ctx->ck_off[e.ls + 1]) RC(ckpt_offload(e.ls + 1, m));
        } else {
          RC(backward(e.ls, e.res, m));
        }
      }
      CU(cudaEventRecord(ctx->ev_pass_b[xi], s));
      if (!e.fwd) {
        bwd_xi[e.ls] = (int)xi;
        // stage ls-2's checkpoints go back into the bank slots B_{ls} just freed
        if (e.ls >= 2 && ctx->ck_off[e.ls - 2]) RC(ckpt_upload(e.ls - 2, ctx->ev_pass_b[xi]));
      }
      if (!e.fwd && ctx->arena_mode) RC(finish_stage_grads(e.ls));  // D2H recorded before the release waits on it
      if (e.last_of_res) {
        CU(cudaEventRecord(ctx->ev_release[e.res], s));
        RC(load_second_part(e.res + 1));
      }
      if (!e.fwd && !ctx->arena_mode) RC(finish_stage_grads(e.ls));
    }
    ctx->last_bwd_host_ns = 0;
    return MOBIUS_OK;
  }
};

int check_ctx(mobius_ctx* ctx) {
  if (!ctx) MOBIUS_FAIL(MOBIUS_EINVAL, "null context");
  if (ctx->poisoned) MOBIUS_FAIL(MOBIUS_ESTATE, "context poisoned by an earlier failure");
  return MOBIUS_OK;
}

template <typename T>
int do_step(mobius_ctx* ctx, const int32_t* tok_dev, int M, float* loss_out) {
  const Shape& sh = ctx->sh;
  StepRunner<T> R;
  R.ctx = ctx;
  R.tok_dev = tok_dev;
  R.M = M;
  R.seq = ctx->step_count + 1;
  R.inv_ntok = 1.0f / ((float)M * sh.mbs * sh.s);
  carve_scratch<T>(sh, ctx->scratch_base, true, R.sc);
  if (ctx->step_count == 0) RC(scratch_zero<T>(R.sc, ctx->s_comp));
  R.acts.resize(std::max(1, ctx->ws_blocks));
  for (int i = 0; i < (int)R.acts.size(); ++i) carve_block_acts<T>(sh, ctx->acts_base + i * ctx->acts_bytes, R.acts[i]);
  ctx->trace.clear();
  ctx->timer.reset();
  if (const char* e = getenv("MOBIUS_TIMING_STRIDE")) ctx->timer.stride = std::max(1, atoi(e));
  ctx->launches_step = 0;
  g_kernel_launches = 0;
  std::memset(&ctx->stats, 0, sizeof(ctx->stats));
  set_kernel_timer((ctx->dist.flags & MOBIUS_FLAG_TIMING) ? &ctx->timer : nullptr);
  int64_t t0 = now_ns();
  CU(cudaEventRecord(ctx->ev_step0, ctx->s_comp));
  CU(cudaMemsetAsync(ctx->loss_dev, 0, sizeof(double), ctx->s_comp));
  if (getenv("MOBIUS_INJECT_CUDA_FAULT"))  // test hook: a (non-sticky) CUDA API failure inside the step
    CU(cudaMemcpyAsync(ctx->tok_dev, nullptr, 4, cudaMemcpyDeviceToDevice, ctx->s_comp));
  int rc = R.run();
  set_kernel_timer(nullptr);
  if (rc) {
    ctx->poisoned = true;
    return rc;
  }
  CU(cudaStreamWaitEvent(ctx->s_comp, ctx->ev_d2h[0], 0));
  CU(cudaEventRecord(ctx->ev_step1, ctx->s_comp));
  CU(cudaMemcpyAsync(ctx->h_loss, ctx->loss_dev, sizeof(double), cudaMemcpyDeviceToHost, ctx->s_comp));
  CU(cudaStreamSynchronize(ctx->s_comp));
  CU(cudaStreamSynchronize(ctx->s_h2d));
  CU(cudaStreamSynchronize(ctx->s_d2h));
  if (ctx->s_p2p) CU(cudaStreamSynchronize(ctx->s_p2p));
  int64_t t_gpu_done = now_ns();
  // The host updates of the stages still in the queue finish while the next
  // step's earlier stages run: every consumer of a stage's new weights (its
  // next swap-in, read_params, destroy) waits for that stage's update, so
  // each step still sees the previous step's parameters.
  // MOBIUS_SYNC_UPDATE=1: wait for all of them here (round-1 behaviour).
  if (ctx->sync_update) drain_updates(ctx);
  int64_t t1 = now_ns();
  const bool has_last = ctx->all.back().owner == ctx->dist.rank;
  *loss_out = has_last ? (float)(*ctx->h_loss * R.inv_ntok) : NAN;
  // stats
  mobius_step_stats& S = ctx->stats;
  S.step_ns = t1 - t0;
  float ms = 0.f;
  cudaEventElapsedTime(&ms, ctx->ev_step0, ctx->ev_step1);
  S.device_step_ns = (int64_t)(ms * 1e6);
  S.h2d_bytes = R.h2d_bytes;
  S.ckpt_d2h_bytes = R.ckpt_d2h;
  S.ckpt_h2d_bytes = R.ckpt_h2d;
  S.n_h2d_copies = R.n_parts;
  S.d2d_bytes = R.d2d_bytes;
  ctx->n_parts_last = R.n_parts;
  if (ctx->dev_tail) ctx->tail_resident = true;  // d_wstage now holds local stage 0's updated weights
  std::vector<double> gbps;
  for (int i = 0; i < R.n_parts; ++i) {
    float pm = 0.f;
    if (ctx->part_bytes[i] > 0 && cudaEventElapsedTime(&pm, ctx->ev_part_a[i], ctx->ev_part_b[i]) == cudaSuccess &&
        pm > 0)
      gbps.push_back(ctx->part_bytes[i] / (pm * 1e-3) / 1e9);
  }
  if (!gbps.empty()) {
    std::sort(gbps.begin(), gbps.end());
    S.h2d_GBps_median = gbps[gbps.size() / 2];
    S.h2d_GBps_max = gbps.back();
  }
  int64_t exposed = 0;
  for (size_t r = 0; r < ctx->loads.size(); ++r) {
    float wm = 0.f;
    if (cudaEventElapsedTime(&wm, ctx->ev_wait_a[r], ctx->ev_wait_b[r]) == cudaSuccess) exposed += (int64_t)(wm * 1e6);
  }
  S.exposed_load_ns = exposed;
  int64_t exposed_ck = 0;
  for (int ls = 0; ls < (int)ctx->mine.size(); ++ls) {
    float wm = 0.f;
    if (ctx->ck_off[ls] && cudaEventElapsedTime(&wm, ctx->ev_ckw_a[ls], ctx->ev_ckw_b[ls]) == cudaSuccess)
      exposed_ck += (int64_t)(wm * 1e6);
  }
  S.exposed_ckpt_ns = exposed_ck;
  for (auto& rec : ctx->timer.recs) {
    float km = 0.f;
    if (cudaEventElapsedTime(&km, rec.a, rec.b) != cudaSuccess) continue;
    // sampled launches scaled by the stride: estimates of the class totals
    int64_t ns = (int64_t)(km * 1e6) * ctx->timer.stride;
    if (rec.cls == KCLS_GEMM) {
      S.gemm_ns += ns;
      S.gemm_flops += rec.flops * ctx->timer.stride;
      S.gemm_launches++;
    } else if (rec.cls == KCLS_ATTN) {
      S.attn_ns += ns;
    } else {
      S.elem_ns += ns;
    }
  }
  S.kernel_launches = ctx->launches_step + g_kernel_launches;
  S.timing_stride = ctx->timer.stride;
  S.arena_bytes = ctx->arena_bytes + ctx->keep_bytes;
  S.ring_bytes = ctx->ring_bytes;
  int64_t pinned = 0;
  for (int ls = 0; ls < (int)ctx->mine.size(); ++ls) {
    pinned += 2 * ctx->all[ctx->mine[ls]].n_params * ctx->esz;
    if (ctx->h_ckpt[ls]) pinned += (int64_t)ctx->max_M * ctx->slot_bytes;
  }
  S.pinned_bytes = pinned;
  S.host_update_ns = ctx->upd_ns;
  S.update_tail_ns = t1 - t_gpu_done + ctx->upd_wait_ns;  // exposed waiting for host updates (here or at issue)
  ctx->upd_wait_ns = 0;
  S.n_local_stages = (int)ctx->mine.size();
  S.recompute = 0;
  for (int ls = 0; ls < (int)ctx->mine.size(); ++ls)
    if (ctx->mine[ls] != ctx->plan.n_stages - 1 && ctx->all[ctx->mine[ls]].n_blocks > 0)
      S.recompute += ctx->all[ctx->mine[ls]].n_blocks - ctx->keep_nb[ls];  // blocks recomputed in backward
  ctx->upd_ns = 0;
  ctx->step_count++;
  return MOBIUS_OK;
}

}  // namespace

// ======================================================================
static int arena_shape(const mobius_model_cfg* c, Shape* sh, int* esz, bool* flash) {
  MOBIUS_CHECK_ARG(c && c->n_layers >= 1 && c->hidden > 0 && c->n_heads > 0 && c->hidden % c->n_heads == 0 &&
                       c->seq_len > 0 && c->vocab > 0 && c->micro_batch > 0 && c->n_layers + 2 <= MOBIUS_MAX_LAYERS,
                   "bad model config");
  *sh = Shape{c->hidden, c->n_heads, c->seq_len, c->micro_batch, c->vocab};
  sh->head_rows = arena_head_rows(*sh);
  sh->no_keep = true;
  *esz = c->dtype == MOBIUS_F32 ? 4 : 2;
  *flash = *esz == 2 && flash_supported(sh->dh(), sh->s);
  return MOBIUS_OK;
}

extern "C" int mobius_arena_layer_sizes(const mobius_model_cfg* c, mobius_layer_profile* out, int* n_out) {
  MOBIUS_CHECK_ARG(out && n_out, "null argument");
  Shape sh;
  int esz;
  bool fl;
  if (int rc = arena_shape(c, &sh, &esz, &fl)) return rc;
  const int64_t slot = al256((int64_t)sh.T() * sh.h * esz);
  const int64_t acts = al256(block_acts_bytes(sh, esz, fl));
  const int Lp = c->n_layers + 2;
  for (int i = 0; i < Lp; ++i) {
    const int64_t np = layer_numel(*c, i);
    const bool block = i > 0 && i < Lp - 1;
    // a stage's footprint is the sum over its layers of these (each region
    // rounded up per layer: >= the runtime's per-stage rounding)
    const BwdFootprint f = bwd_footprint(np, esz, block ? 1 : 0, i == 0, acts, slot);
    mobius_layer_profile& p = out[i];
    std::memset(&p, 0, sizeof(p));
    p.mem_fwd = al256(np * esz);
    p.mem_bwd = f.total;
    p.xfer_fwd = p.xfer_bwd = np * esz;
    p.act_out = (int64_t)sh.T() * sh.h * esz;
  }
  *n_out = Lp;
  return MOBIUS_OK;
}

extern "C" int mobius_arena_fixed_bytes(const mobius_model_cfg* c, int n_microbatches, int n_local_stages, int flags,
                                        int64_t* bytes) {
  MOBIUS_CHECK_ARG(bytes && n_microbatches >= 1 && n_local_stages >= 1, "bad arguments");
  Shape sh;
  int esz;
  bool fl;
  if (int rc = arena_shape(c, &sh, &esz, &fl)) return rc;
  const int64_t slot = al256((int64_t)sh.T() * sh.h * esz);
  const FixedLayout f = fixed_layout(sh, esz, fl, n_microbatches, n_local_stages, 0, 0, true,
                                     (flags & MOBIUS_FLAG_CKPT_OFFLOAD) != 0, slot, 0);
  *bytes = f.end;
  return MOBIUS_OK;
}

extern "C" int mobius_create(const mobius_model_cfg* cfg, const mobius_plan_t* plan, const mobius_dist* dist,
                             const float* init_params, uint64_t seed, mobius_ctx** out) {
  MOBIUS_CHECK_ARG(cfg && plan && dist && out, "null argument");
  *out = nullptr;
  const mobius_model_cfg& c = *cfg;
  MOBIUS_CHECK_ARG(c.dtype == MOBIUS_BF16 || c.dtype == MOBIUS_F32, "bad dtype");
  MOBIUS_CHECK_ARG(c.n_layers >= 1 && c.hidden % 64 == 0 && c.n_heads > 0 && c.hidden % c.n_heads == 0,
                   "hidden must be a multiple of 64 and of n_heads");
  const int dh = c.hidden / c.n_heads;
  if (c.dtype == MOBIUS_BF16) {
    MOBIUS_CHECK_ARG(dh == 64 || dh == 128, "bf16 path needs head_dim 64 or 128 (got %d)", dh);
    MOBIUS_CHECK_ARG(c.seq_len % 8 == 0 && c.vocab % 8 == 0, "seq_len and vocab must be multiples of 8");
  }
  const int Lp = c.n_layers + 2;
  MOBIUS_CHECK_ARG(plan->n_layers == Lp || plan->n_layers == 0, "plan has %d layers, model %d", plan->n_layers, Lp);
  MOBIUS_CHECK_ARG(plan->n_stages >= 1 && plan->n_stages <= Lp, "bad stage count");
  MOBIUS_CHECK_ARG(plan->n_gpus == dist->world && dist->world >= 1 && dist->rank >= 0 && dist->rank < dist->world,
                   "plan n_gpus %d != world %d", plan->n_gpus, dist->world);
  MOBIUS_CHECK_ARG(plan->stage_first_layer[0] == 0 && plan->stage_first_layer[plan->n_stages] == Lp,
                   "stage boundaries must cover all %d profile layers", Lp);
  for (int j = 0; j < plan->n_stages; ++j) {
    MOBIUS_CHECK_ARG(plan->stage_first_layer[j + 1] > plan->stage_first_layer[j], "empty stage %d", j);
    MOBIUS_CHECK_ARG(plan->stage_gpu[j] >= 0 && plan->stage_gpu[j] < dist->world, "bad stage_gpu");
    MOBIUS_CHECK_ARG(plan->stage_gpu[j] == plan->stage_gpu[j % plan->n_gpus], "stage_gpu must be round-robin");
  }

  std::unique_ptr<mobius_ctx> ctx(new mobius_ctx());
  ctx->cfg = c;
  ctx->plan = *plan;
  ctx->plan.n_layers = Lp;
  ctx->dist = *dist;
  ctx->sh = Shape{c.hidden, c.n_heads, c.seq_len, c.micro_batch, c.vocab};
  ctx->esz = c.dtype == MOBIUS_F32 ? 4 : 2;
  const int esz = ctx->esz;
  mobius_ctx* raw = ctx.get();
  (void)raw;

  // stages
  const int K = plan->n_stages;
  ctx->all.resize(K);
  std::vector<int> count(dist->world, 0);
  int64_t poff = 0;
  for (int j = 0; j < K; ++j) {
    StageDesc& st = ctx->all[j];
    st.j = j;
    st.first = plan->stage_first_layer[j];
    st.last = plan->stage_first_layer[j + 1];
    st.param_off = poff;
    int64_t o = 0;
    for (int li = st.first; li < st.last; ++li) {
      st.layer_off.push_back(o);
      o += layer_numel(c, li);
      if (li == 0) st.has_embed = true;
      else if (li == Lp - 1) st.has_head = true;
      else st.n_blocks++;
    }
    st.n_params = o;
    poff += o;
    st.owner = plan->stage_gpu[j];
    st.ord = count[st.owner]++;
    if (st.owner == dist->rank) ctx->mine.push_back(j);
  }
  MOBIUS_CHECK_ARG(!ctx->mine.empty(), "rank %d owns no stage", dist->rank);
  const int n = (int)ctx->mine.size();

  const bool arena = (dist->flags & MOBIUS_FLAG_ARENA_CAP) != 0;
  const bool offload = (dist->flags & MOBIUS_FLAG_CKPT_OFFLOAD) != 0;
  MOBIUS_CHECK_ARG(!offload || dist->world == 1, "MOBIUS_FLAG_CKPT_OFFLOAD needs world size 1 (banked slots are "
                                                 "written by a peer at N > 1)");
  MOBIUS_CHECK_ARG(!(arena && (dist->flags & MOBIUS_FLAG_DEVICE_TAIL_UPDATE)),
                   "MOBIUS_FLAG_ARENA_CAP excludes MOBIUS_FLAG_DEVICE_TAIL_UPDATE (its optimizer state is outside "
                   "the capped memory)");
  MOBIUS_CHECK_ARG(!arena || plan->hbm_cap_bytes > 0, "MOBIUS_FLAG_ARENA_CAP needs a cap");
  ctx->arena_mode = arena;
  ctx->offload = offload;
  if (arena) {
    ctx->sh.head_rows = arena_head_rows(ctx->sh);
    ctx->sh.no_keep = true;
  }

  // per-microbatch sizes
  const Shape& sh = ctx->sh;
  const int M = plan->n_microbatches > 0 ? plan->n_microbatches : dist->world;
  ctx->max_M = M;
  ctx->slot_bytes = al256((int64_t)sh.T() * sh.h * esz);
  const bool fl = esz == 2 && flash_supported(sh.dh(), sh.s);
  ctx->acts_bytes = al256(block_acts_bytes(sh, esz, fl));
  ctx->keep_compact = fl && !getenv("MOBIUS_KEEP_FULL");
  ctx->keep_acts_bytes = al256(block_acts_bytes(sh, esz, fl, ctx->keep_compact));

  // ring: cap G (plan) or double-buffer default
  int64_t max_stage = 0, max_params = 0;
  for (int ls = 0; ls < n; ++ls) {
    const StageDesc& st = ctx->all[ctx->mine[ls]];
    max_stage = std::max(max_stage, st.n_params * esz);
    max_params = std::max(max_params, st.n_params);
    ctx->max_blocks = std::max(ctx->max_blocks, st.n_blocks);
  }
  int64_t G = plan->hbm_cap_bytes > 0 ? (plan->hbm_cap_bytes & ~int64_t(255)) : 2 * al256(max_stage);
  ctx->ring_bytes = G;

  // residences: fwd loads ascending, bwd reloads descending except the last
  // (which stays resident: its forward residence is its backward one)
  auto footprint = [&](int k, bool bwd) -> int64_t {
    const StageDesc& st = ctx->all[ctx->mine[k]];
    if (!arena || !bwd) return st.n_params * esz;
    return bwd_footprint(st.n_params, esz, st.n_blocks, st.has_embed, ctx->acts_bytes, ctx->slot_bytes).total;
  };
  ctx->res_f.assign(n, -1);
  ctx->res_b.assign(n, -1);
  for (int k = 0; k < n; ++k) {
    ctx->res_f[k] = (int)ctx->loads.size();
    const bool last = k == n - 1;
    ctx->loads.push_back({k, 0, 0, footprint(k, last), ctx->all[ctx->mine[k]].n_params * esz, last});
  }
  ctx->res_b[n - 1] = ctx->res_f[n - 1];
  for (int k = n - 2; k >= 0; --k) {
    ctx->res_b[k] = (int)ctx->loads.size();
    ctx->loads.push_back({k, 0, 0, footprint(k, true), ctx->all[ctx->mine[k]].n_params * esz, true});
  }
  int64_t max_fp = 0;
  for (const Load& L : ctx->loads) max_fp = std::max(max_fp, L.bytes);
  if (max_fp > G)
    MOBIUS_FAIL(MOBIUS_EINFEASIBLE, "stage %s of %lld bytes exceeds the cap %lld", arena ? "footprint" : "",
                (long long)max_fp, (long long)G);
  for (size_t r = 0; r < ctx->loads.size(); ++r) {
    Load& L = ctx->loads[r];
    L.end = (int)(r % 2);
    L.base = L.end == 0 ? 0 : ((G - L.bytes) & ~int64_t(255));
    if (arena && L.bwd && L.end == 1) {
      const StageDesc& st = ctx->all[ctx->mine[L.stage_local]];
      L.wofs = bwd_footprint(st.n_params, esz, st.n_blocks, st.has_embed, ctx->acts_bytes, ctx->slot_bytes, true).w;
    }
  }

  // arena layout behind the ring
  const FixedLayout FL = fixed_layout(sh, esz, fl, M, n, ctx->max_blocks, max_params, arena, offload,
                                      ctx->slot_bytes, G);
  ctx->xs_fixed = FL.xs_slots;
  int64_t o_gacc = FL.gacc;
  int64_t o_gstage = FL.gstage;
  ctx->off_ckpt = FL.ckpt;
  ctx->off_gslot = FL.gslot;
  ctx->off_fflag = FL.fflag;
  ctx->off_bflag = FL.bflag;
  ctx->off_pf = FL.pf;
  int64_t o_xs = FL.xs;
  int64_t o_scr = FL.scr;
  int64_t o_tok = FL.tok;
  int64_t o_loss = FL.loss;
  int64_t o_bad = FL.bad;
  const int64_t o_acts = FL.acts;
  (void)o_xs;

  int cu_dev = dist->device;
  {
    mobius_ctx* ctxp = ctx.get();
    mobius_ctx* ctx = ctxp;  // for CU()
    CU(cudaSetDevice(cu_dev));
    // kept activations (reading #17: keep instead of recompute when they fit):
    // whole local stages, latest first, else a stage's last blocks, within the
    // free HBM minus a margin.  The recompute workspace (acts, full layout) is
    // then sized by what is still recomputed - the last stage (forward folded
    // into backward) and the non-kept blocks - instead of the largest stage;
    // the two are solved together (the workspace only grows, a few rounds).
    ctx->keep_off.assign(n, -1);
    ctx->keep_nb.assign(n, 0);
    const int64_t dev_tail_bytes = (dist->flags & MOBIUS_FLAG_DEVICE_TAIL_UPDATE) && n > 0
        ? al256(ctx->all[ctx->mine[0]].n_params * 4) * 3 + al256(ctx->all[ctx->mine[0]].n_params * esz) : 0;
    int ws = arena ? 1 : std::max(1, ctx->max_blocks);  // arena: the recompute sets live in the residences
    int64_t keep_total = 0;
    if ((dist->flags & MOBIUS_FLAG_KEEP_ACTS) && !arena) {
      size_t fr = 0, tot = 0;
      CU(cudaMemGetInfo(&fr, &tot));
      // margin for what is allocated after create (Stream-K workspaces, the
      // caller's buffers: tens of MB); MOBIUS_KEEP_MARGIN_GIB overrides the
      // default 2.5 GiB (6 GiB cost one more recomputed block at 1.5B / mbs 32)
      double margin_gib = 2.5;
      if (const char* e = getenv("MOBIUS_KEEP_MARGIN_GIB")) margin_gib = std::max(0.5, atof(e));
      const int64_t entry = ctx->keep_acts_bytes + ctx->slot_bytes;
      ws = 1;
      for (int k = 0; k < n; ++k)
        if (ctx->all[ctx->mine[k]].j == plan->n_stages - 1) ws = std::max(ws, ctx->all[ctx->mine[k]].n_blocks);
      for (int round = 0; round < 8; ++round) {
        int64_t budget = (int64_t)fr - o_acts - al256(ctx->acts_bytes * ws) - dev_tail_bytes -
                         (int64_t)(margin_gib * (1LL << 30));
        if (const char* e = getenv("MOBIUS_KEEP_GIB"))
          budget = std::min<int64_t>(budget, (int64_t)(atof(e) * (1LL << 30)));
        int64_t koff = 0;
        int need_ws = ws;
        for (int k = n - 1; k >= 0; --k) {
          const StageDesc& st = ctx->all[ctx->mine[k]];
          ctx->keep_off[k] = -1;
          ctx->keep_nb[k] = 0;
          if (st.j == plan->n_stages - 1 || st.n_blocks == 0) continue;  // last stage: F is folded into B
          // whole stage if it fits, else its last blocks (the rest is recomputed)
          int nb = st.n_blocks;
          while (nb > 0 && koff + al256((int64_t)M * nb * entry) > budget) --nb;
          need_ws = std::max(need_ws, st.n_blocks - nb);
          if (nb == 0) continue;
          ctx->keep_off[k] = koff;
          ctx->keep_nb[k] = nb;
          koff += al256((int64_t)M * nb * entry);
        }
        keep_total = koff;
        if (need_ws <= ws) break;
        ws = need_ws;
      }
    }
    ctx->ws_blocks = ws;
    ctx->arena_bytes = arena ? FL.end : o_acts + al256(ctx->acts_bytes * ws);
    CU(cudaMalloc(&ctx->arena, ctx->arena_bytes));
    if (!arena) CU(cudaMemset(ctx->arena + o_gacc, 0, max_params * 4));
    ctx->ring = ctx->arena;
    ctx->dev_tail = (dist->flags & MOBIUS_FLAG_DEVICE_TAIL_UPDATE) && n > 0;
    if (ctx->dev_tail) {  // before the keep pool takes the free HBM
      const int64_t np0 = ctx->all[ctx->mine[0]].n_params;
      ctx->d_opt_stride = al256(np0 * 4) / 4;
      CU(cudaMalloc(&ctx->d_opt, ctx->d_opt_stride * 4 * 3));
      CU(cudaMalloc(&ctx->d_wstage, al256(np0 * esz)));
    }
    if (keep_total > 0) {
      CU(cudaMalloc(&ctx->keep_pool, keep_total));
      ctx->keep_bytes = keep_total;
    }
    ctx->grad_acc = arena ? nullptr : reinterpret_cast<float*>(ctx->arena + o_gacc);  // arena: per residence
    ctx->grad_stage = arena ? nullptr : ctx->arena + o_gstage;
    ctx->ckpt = ctx->arena + ctx->off_ckpt;
    ctx->gslot = ctx->arena + ctx->off_gslot;
    ctx->fflag = reinterpret_cast<int*>(ctx->arena + ctx->off_fflag);
    ctx->bflag = reinterpret_cast<int*>(ctx->arena + ctx->off_bflag);
    ctx->acts_base = ctx->arena + o_acts;
    ctx->xs_base = ctx->arena + o_xs;
    ctx->scratch_base = ctx->arena + o_scr;
    ctx->tok_dev = ctx->arena + o_tok;
    ctx->loss_dev = reinterpret_cast<double*>(ctx->arena + o_loss);
    ctx->bad_tok_dev = reinterpret_cast<int*>(ctx->arena + o_bad);
    CU(cudaMemset(ctx->fflag, 0, (int64_t)n * M * 4));
    CU(cudaMemset(ctx->bflag, 0, (int64_t)n * M * 4));
    ctx->pf_base = reinterpret_cast<int*>(ctx->arena + ctx->off_pf);
    CU(cudaMemset(ctx->pf_base, 0, (1 + 4 * (int64_t)n) * 4));

    // streams: H2D prefetch gets the highest priority
    int lo = 0, hi = 0;
    CU(cudaDeviceGetStreamPriorityRange(&lo, &hi));
    CU(cudaStreamCreateWithPriority(&ctx->s_comp, cudaStreamNonBlocking, lo));
    CU(cudaStreamCreateWithPriority(&ctx->s_h2d, cudaStreamNonBlocking, hi));
    CU(cudaStreamCreateWithPriority(&ctx->s_d2h, cudaStreamNonBlocking, lo));
    const int R = (int)ctx->loads.size();
    auto mk = [&](std::vector<cudaEvent_t>& v, int cnt, unsigned flags) -> int {
      v.resize(cnt);
      for (auto& e : v) CU(cudaEventCreateWithFlags(&e, flags));
      return MOBIUS_OK;
    };
    RC(mk(ctx->ev_release, R, cudaEventDisableTiming));
    RC(mk(ctx->ev_loaded, R, cudaEventDisableTiming));
    RC(mk(ctx->ev_part_a, 2 * R + 2, cudaEventDefault));
    RC(mk(ctx->ev_part_b, 2 * R + 2, cudaEventDefault));
    ctx->part_bytes.assign(2 * R + 2, 0);
    RC(mk(ctx->ev_gready, n, cudaEventDisableTiming));
    RC(mk(ctx->ev_d2h, n, cudaEventDisableTiming));
    RC(mk(ctx->ev_wait_a, R, cudaEventDefault));
    RC(mk(ctx->ev_pass_a, 2 * n, cudaEventDefault));
    RC(mk(ctx->ev_pass_b, 2 * n, cudaEventDefault));
    RC(mk(ctx->ev_off_a, n, cudaEventDefault));
    RC(mk(ctx->ev_off_b, n, cudaEventDefault));
    ctx->part_stage.assign(2 * R + 2, 0);
    ctx->part_d2d.assign(2 * R + 2, 0);
    RC(mk(ctx->ev_wait_b, R, cudaEventDefault));
    CU(cudaEventCreate(&ctx->ev_step0));
    CU(cudaEventCreate(&ctx->ev_step1));
    for (int k = 0; k < n; ++k) CU(cudaEventRecord(ctx->ev_d2h[k], ctx->s_d2h));
    // checkpoint offload: stage k (1 <= k <= n-3) has its input slot reused
    // by stage k+2's input, so its checkpoints round-trip through DRAM
    ctx->ck_off.assign(n, 0);
    ctx->h_ckpt.assign(n, nullptr);
    if (offload) {
      CU(cudaStreamCreateWithPriority(&ctx->s_ckup, cudaStreamNonBlocking, hi));
      RC(mk(ctx->ev_ckoff, 2 * M, cudaEventDisableTiming));
      RC(mk(ctx->ev_ckprod, M, cudaEventDisableTiming));
      RC(mk(ctx->ev_ckup, n, cudaEventDisableTiming));
      RC(mk(ctx->ev_ck_a, 2 * n, cudaEventDefault));
      RC(mk(ctx->ev_ck_b, 2 * n, cudaEventDefault));
      RC(mk(ctx->ev_ckw_a, n, cudaEventDefault));
      RC(mk(ctx->ev_ckw_b, n, cudaEventDefault));
      CU(cudaEventCreateWithFlags(&ctx->ev_fwd_off, cudaEventDisableTiming));
      CU(cudaEventRecord(ctx->ev_fwd_off, ctx->s_d2h));
      for (int k = 1; k + 2 < n; ++k) {
        ctx->ck_off[k] = 1;
        CU(cudaHostAlloc(&ctx->h_ckpt[k], (size_t)M * ctx->slot_bytes, cudaHostAllocDefault));
      }
    }

    // host stage store
    unsigned hw = std::thread::hardware_concurrency();
    int nthreads = std::max(1, (int)(hw ? hw : 4) / dist->world);
    ctx->pool.reset(new ThreadPool(nthreads));
    ctx->h_weights.resize(n);
    ctx->h_grads.resize(n);
    ctx->upd_done.assign(n, 0);
    ctx->sync_update = getenv("MOBIUS_SYNC_UPDATE") != nullptr;
    ctx->h_master.resize(n);
    ctx->h_m.resize(n);
    ctx->h_v.resize(n);
    for (int k = 0; k < n; ++k) {
      const StageDesc& st = ctx->all[ctx->mine[k]];
      const int64_t np = st.n_params;
      CU(cudaHostAlloc(&ctx->h_weights[k], al256(np * esz), cudaHostAllocDefault));
      CU(cudaHostAlloc(&ctx->h_grads[k], al256(np * esz), cudaHostAllocDefault));
      // 64-byte aligned so the AVX-512 update can use non-temporal stores
      const size_t nb = (size_t)((np * 4 + 63) / 64 * 64);
      float* mst = (float*)std::aligned_alloc(64, nb);
      float* mm = (float*)std::aligned_alloc(64, nb);
      float* vv = (float*)std::aligned_alloc(64, nb);
      if (!mst || !mm || !vv) MOBIUS_FAIL(MOBIUS_ENOMEM, "host optimizer state (%lld params)", (long long)np);
      ctx->h_master[k] = mst;
      ctx->h_m[k] = mm;
      ctx->h_v[k] = vv;
      // first touch from the pool threads (NUMA-local pages)
      const int64_t chunk = 1 << 20;
      const int tasks = (int)((np + chunk - 1) / chunk);
      ctx->pool->parallel_for(tasks, [&](int t) {
        int64_t b = (int64_t)t * chunk, e = std::min(np, b + chunk);
        if (init_params)
          std::memcpy(mst + b, init_params + st.param_off + b, (e - b) * 4);
        std::memset(mm + b, 0, (e - b) * 4);
        std::memset(vv + b, 0, (e - b) * 4);
      });
      if (!init_params) {
        g_init_pool = ctx->pool.get();
        seeded_stage_init(c, st, mst, seed);
        g_init_pool = nullptr;
      }
      ctx->pool->parallel_for(tasks, [&](int t) {
        int64_t b = (int64_t)t * chunk, e = std::min(np, b + chunk);
        if (esz == 2) {
          uint16_t* w = (uint16_t*)ctx->h_weights[k];
          for (int64_t i = b; i < e; ++i) w[i] = f32_to_bf16_rne(mst[i]);
        } else {
          std::memcpy((float*)ctx->h_weights[k] + b, mst + b, (e - b) * 4);
        }
      });
    }
    if (ctx->dev_tail) {  // stage 0's optimizer state moves to HBM (m = v = 0)
      const int64_t np0 = ctx->all[ctx->mine[0]].n_params;
      CU(cudaMemcpy(ctx->d_opt, ctx->h_master[0], np0 * 4, cudaMemcpyHostToDevice));
      CU(cudaMemset(ctx->d_opt + ctx->d_opt_stride, 0, ctx->d_opt_stride * 4 * 2));
    }
    CU(cudaHostAlloc(&ctx->h_loss, sizeof(double), cudaHostAllocDefault));
    ctx->h_tokens_cap = (int64_t)M * sh.mbs * (sh.s + 1);
    CU(cudaHostAlloc(&ctx->h_tokens, ctx->h_tokens_cap * 4, cudaHostAllocDefault));
    CU(cudaHostAlloc(&ctx->h_bad_tok, sizeof(int), cudaHostAllocDefault));
    ctx->peer_base.assign(dist->world, nullptr);
    ctx->connected = dist->world == 1;
    CU(cudaDeviceSynchronize());
    ctx->upd_thread = std::thread(update_worker, ctxp);  // last: nothing after it can fail
  }
  *out = ctx.release();
  return MOBIUS_OK;
}

struct ExportBlob {
  uint32_t magic;
  int32_t rank;
  uint64_t plan_digest;  // every rank must run the identical plan (SPMD contract)
  cudaIpcMemHandle_t handle;
  int64_t off_ckpt, off_gslot, off_fflag, off_bflag, slot_bytes;
  int32_t n_local, M;
  int64_t off_pf;
};

static uint64_t plan_digest(const mobius_ctx* ctx) {
  uint64_t h = 1469598103934665603ull;  // FNV-1a over the plan and model shape
  auto mix = [&](int64_t v) {
    for (int i = 0; i < 8; ++i) {
      h ^= (uint64_t)((v >> (8 * i)) & 0xff);
      h *= 1099511628211ull;
    }
  };
  const mobius_plan_t& p = ctx->plan;
  mix(p.n_stages);
  mix(p.n_gpus);
  mix(ctx->max_M);
  for (int j = 0; j <= p.n_stages; ++j) mix(p.stage_first_layer[j]);
  for (int j = 0; j < p.n_stages; ++j) mix(p.stage_gpu[j]);
  const mobius_model_cfg& c = ctx->cfg;
  mix(c.n_layers);
  mix(c.hidden);
  mix(c.n_heads);
  mix(c.seq_len);
  mix(c.vocab);
  mix(c.micro_batch);
  mix(c.dtype);
  return h;
}

extern "C" int mobius_dist_export(mobius_ctx* ctx, void* buf, size_t cap, size_t* len) {
  int rc = check_ctx(ctx);
  if (rc) return rc;
  MOBIUS_CHECK_ARG(buf && len && cap >= sizeof(ExportBlob), "export buffer too small");
  ExportBlob b;
  std::memset(&b, 0, sizeof(b));
  b.magic = 0x4d4f4249;
  b.rank = ctx->dist.rank;
  b.plan_digest = plan_digest(ctx);
  CU(cudaSetDevice(ctx->dist.device));
  CU(cudaIpcGetMemHandle(&b.handle, ctx->arena));
  b.off_ckpt = ctx->off_ckpt;
  b.off_gslot = ctx->off_gslot;
  b.off_fflag = ctx->off_fflag;
  b.off_bflag = ctx->off_bflag;
  b.off_pf = ctx->off_pf;
  b.slot_bytes = ctx->slot_bytes;
  b.n_local = (int)ctx->mine.size();
  b.M = ctx->max_M;
  std::memcpy(buf, &b, sizeof(b));
  *len = sizeof(b);
  return MOBIUS_OK;
}

extern "C" int mobius_dist_connect(mobius_ctx* ctx, const void* all, size_t blob_len) {
  int rc = check_ctx(ctx);
  if (rc) return rc;
  MOBIUS_CHECK_ARG(all && blob_len >= sizeof(ExportBlob), "bad blobs");
  const int W = ctx->dist.world;
  ctx->peers.resize(W);
  ctx->p2p_copy.assign(W, 0);
  CU(cudaSetDevice(ctx->dist.device));
  for (int r = 0; r < W; ++r) {
    ExportBlob b;
    std::memcpy(&b, (const char*)all + r * blob_len, sizeof(b));
    MOBIUS_CHECK_ARG(b.magic == 0x4d4f4249 && b.rank == r, "blob %d is not a mobius export", r);
    MOBIUS_CHECK_ARG(b.plan_digest == plan_digest(ctx), "rank %d runs a different plan / config than rank %d", r,
                     ctx->dist.rank);
    PeerInfo& p = ctx->peers[r];
    p.rank = r;
    p.handle = b.handle;
    p.off_ckpt = b.off_ckpt;
    p.off_gslot = b.off_gslot;
    p.off_fflag = b.off_fflag;
    p.off_bflag = b.off_bflag;
    p.off_pf = b.off_pf;
    p.slot_bytes = b.slot_bytes;
    p.n_local = b.n_local;
    p.M = b.M;
    if (r == ctx->dist.rank) continue;
    // only neighbours in the stage chain need a mapping
    bool neighbour = false;
    for (int j = 0; j + 1 < ctx->plan.n_stages; ++j) {
      int a = ctx->all[j].owner, c = ctx->all[j + 1].owner;
      if ((a == ctx->dist.rank && c == r) || (c == ctx->dist.rank && a == r)) neighbour = true;
    }
    if (!ctx->pf_group.empty() && ctx->pf_group[r] == ctx->pf_group[ctx->dist.rank]) neighbour = true;
    if (!neighbour) continue;
    void* ptr = nullptr;
    CU(cudaIpcOpenMemHandle(&ptr, b.handle, cudaIpcMemLazyEnablePeerAccess));
    ctx->peer_base[r] = (uint8_t*)ptr;
    cudaPointerAttributes pa;
    CU(cudaPointerGetAttributes(&pa, ptr));
    const char* direct = getenv("MOBIUS_P2P_DIRECT");
    const char* copy = getenv("MOBIUS_P2P_COPY");
    ctx->p2p_copy[r] = (copy && copy[0] == '1') || (pa.device != ctx->dist.device && !(direct && direct[0] == '1'));
  }
  bool any_copy = false;
  for (char c : ctx->p2p_copy) any_copy |= c != 0;
  if (any_copy && !ctx->send_stage) {
    CU(cudaMalloc(&ctx->send_stage, 2 * ctx->slot_bytes));
    CU(cudaStreamCreateWithFlags(&ctx->s_p2p, cudaStreamNonBlocking));
    for (auto* e : {&ctx->ev_send[0], &ctx->ev_send[1], &ctx->ev_sprod}) CU(cudaEventCreateWithFlags(e, cudaEventDisableTiming));
    CU(cudaEventRecord(ctx->ev_send[0], ctx->s_p2p));
    CU(cudaEventRecord(ctx->ev_send[1], ctx->s_p2p));
  }
  ctx->connected = true;
  return MOBIUS_OK;
}

extern "C" int mobius_set_prefetch_groups(mobius_ctx* ctx, const int* group, int world) {
  int rc = check_ctx(ctx);
  if (rc) return rc;
  MOBIUS_CHECK_ARG(group && world == ctx->dist.world, "group[world] required (world %d)", ctx->dist.world);
  MOBIUS_CHECK_ARG(ctx->peers.empty(), "call mobius_set_prefetch_groups before mobius_dist_connect");
  const mobius_plan_t& P = ctx->plan;
  const int K = P.n_stages, M = ctx->max_M;
  // unit-time plan schedule (a stage's time = its layer count, free
  // transfers): the planned start of every stage pass, a linear extension
  // of the step's dependency graph, so ordering loads by it adds no cycle
  std::vector<mobius_layer_profile> unit(P.n_layers);
  for (auto& l : unit) {
    std::memset(&l, 0, sizeof(l));
    l.t_fwd_ns = l.t_bwd_ns = 1;
    l.mem_fwd = l.mem_bwd = 1;
  }
  std::vector<int> sizes(K);
  for (int j = 0; j < K; ++j) sizes[j] = P.stage_first_layer[j + 1] - P.stage_first_layer[j];
  std::vector<int64_t> tf((size_t)K * M), tb((size_t)K * M);
  int64_t mk = 0;
  rc = mobius_plan_cost(unit.data(), P.n_layers, sizes.data(), K, world, INT64_MAX / 4, M, 0, 0, &mk, tf.data(),
                        tb.data());
  if (rc) return rc;
  struct PL {
    int64_t key;
    int rank, r;
  };
  std::vector<PL> chain;
  const int me = ctx->dist.rank;
  int leader = world;
  for (int g = 0; g < world; ++g) {
    if (group[g] != group[me]) continue;
    leader = std::min(leader, g);
    std::vector<int> st;
    for (int j = 0; j < K; ++j)
      if (ctx->all[j].owner == g) st.push_back(j);
    const int n = (int)st.size();
    int r = 0;
    for (int k = 0; k < n; ++k) chain.push_back({tf[(size_t)st[k] * M], g, r++});      // forward loads
    for (int k = n - 2; k >= 0; --k) chain.push_back({tb[(size_t)st[k] * M], g, r++});  // backward reloads
  }
  std::stable_sort(chain.begin(), chain.end(), [](const PL& a, const PL& b) {
    if (a.key != b.key) return a.key < b.key;
    if (a.rank != b.rank) return a.rank < b.rank;
    return a.r < b.r;
  });
  const int R = (int)ctx->loads.size();
  ctx->pf_pred_rank.assign(R, -1);
  ctx->pf_pred_load.assign(R, -1);
  for (size_t i = 0; i < chain.size(); ++i) {
    if (chain[i].rank != me) continue;
    MOBIUS_CHECK_ARG(chain[i].r < R, "prefetch chain: load count mismatch");
    if (i > 0 && chain[i - 1].rank != me) {
      ctx->pf_pred_rank[chain[i].r] = chain[i - 1].rank;
      ctx->pf_pred_load[chain[i].r] = chain[i - 1].r;
    }
  }
  ctx->pf_group.assign(group, group + world);
  ctx->pf_leader = leader;
  return MOBIUS_OK;
}

extern "C" int mobius_read_prefetch_tickets(mobius_ctx* ctx, int32_t* out, size_t cap, size_t* n) {
  int rc = check_ctx(ctx);
  if (rc) return rc;
  MOBIUS_CHECK_ARG(out && n, "null argument");
  const int R = (int)ctx->loads.size();
  *n = R;
  if (ctx->pf_group.empty()) MOBIUS_FAIL(MOBIUS_ESTATE, "no prefetch chain (mobius_set_prefetch_groups)");
  CU(cudaSetDevice(ctx->dist.device));
  std::vector<int32_t> t(R);
  CU(cudaMemcpy(t.data(), ctx->pf_base + 1 + R, R * 4, cudaMemcpyDeviceToHost));
  std::memcpy(out, t.data(), std::min(cap, (size_t)R) * 4);
  return MOBIUS_OK;
}

static int step_common(mobius_ctx* ctx, const int32_t* tok_dev, int M, float* loss_out) {
  if (ctx->cfg.dtype == MOBIUS_F32) return do_step<float>(ctx, tok_dev, M, loss_out);
  return do_step<bf16>(ctx, tok_dev, M, loss_out);
}

extern "C" int mobius_step(mobius_ctx* ctx, const int32_t* tokens, int M, float* loss_out) {
  int rc = check_ctx(ctx);
  if (rc) return rc;
  MOBIUS_CHECK_ARG(tokens && loss_out && M >= 1, "bad arguments");
  MOBIUS_CHECK_ARG(M == ctx->max_M, "n_microbatches %d != plan's %d", M, ctx->max_M);
  if (!ctx->connected) MOBIUS_FAIL(MOBIUS_ESTATE, "world > 1: call mobius_dist_connect first");
  CU(cudaSetDevice(ctx->dist.device));
  const int64_t n = (int64_t)M * ctx->sh.mbs * (ctx->sh.s + 1);
  // token ids index wte rows and the logits (embedding gather / scatter, CE):
  // an id outside [0, V) is rejected before anything runs
  const int32_t V = ctx->cfg.vocab;
  for (int64_t i = 0; i < n; ++i)
    if ((uint32_t)tokens[i] >= (uint32_t)V)
      MOBIUS_FAIL(MOBIUS_EINVAL, "token %lld = %d outside [0, %d)", (long long)i, tokens[i], V);
  std::memcpy(ctx->h_tokens, tokens, n * 4);
  CU(cudaMemcpyAsync(ctx->tok_dev, ctx->h_tokens, n * 4, cudaMemcpyHostToDevice, ctx->s_comp));
  return step_common(ctx, reinterpret_cast<const int32_t*>(ctx->tok_dev), M, loss_out);
}

extern "C" int mobius_step_device(mobius_ctx* ctx, const int32_t* tokens_dev, int M, float* loss_out) {
  int rc = check_ctx(ctx);
  if (rc) return rc;
  MOBIUS_CHECK_ARG(tokens_dev && loss_out && M == ctx->max_M, "bad arguments");
  if (!ctx->connected) MOBIUS_FAIL(MOBIUS_ESTATE, "world > 1: call mobius_dist_connect first");
  CU(cudaSetDevice(ctx->dist.device));
  // copy into the context's token buffer while counting ids outside [0, V)
  // (one small kernel + a sync before the step: a bad id would otherwise
  // scatter into arbitrary arena memory in the embedding backward)
  const int64_t n = (int64_t)M * ctx->sh.mbs * (ctx->sh.s + 1);
  RC(tokens_check_copy(tokens_dev, reinterpret_cast<int32_t*>(ctx->tok_dev), n, ctx->cfg.vocab, ctx->bad_tok_dev,
                       ctx->s_comp));
  CU(cudaMemcpyAsync(ctx->h_bad_tok, ctx->bad_tok_dev, sizeof(int), cudaMemcpyDeviceToHost, ctx->s_comp));
  CU(cudaStreamSynchronize(ctx->s_comp));
  if (*ctx->h_bad_tok) MOBIUS_FAIL(MOBIUS_EINVAL, "%d token ids outside [0, %d)", *ctx->h_bad_tok, ctx->cfg.vocab);
  return step_common(ctx, reinterpret_cast<const int32_t*>(ctx->tok_dev), M, loss_out);
}

extern "C" int mobius_read_grads(mobius_ctx* ctx, float* out, size_t n) {
  int rc = check_ctx(ctx);
  if (rc) return rc;
  drain_updates(ctx);  // the landing buffers are stable once their updates have read them
  MOBIUS_CHECK_ARG(out, "null out");
  for (int ls = 0; ls < (int)ctx->mine.size(); ++ls) {
    const StageDesc& st = ctx->all[ctx->mine[ls]];
    MOBIUS_CHECK_ARG((size_t)(st.param_off + st.n_params) <= n, "output too small");
    const void* src = ctx->h_grads[ls];
    std::vector<uint8_t> tmp;
    if (ctx->dev_tail && ls == 0) {  // never offloaded: the staging buffer still holds it (last stage in backward)
      tmp.resize(st.n_params * ctx->esz);
      if (cudaMemcpy(tmp.data(), ctx->grad_stage, tmp.size(), cudaMemcpyDeviceToHost) != cudaSuccess)
        MOBIUS_FAIL(MOBIUS_ECUDA, "read_grads: device copy");
      src = tmp.data();
    }
    if (ctx->esz == 2) {
      const uint16_t* g = (const uint16_t*)src;
      for (int64_t i = 0; i < st.n_params; ++i) out[st.param_off + i] = bf16_to_f32(g[i]);
    } else {
      std::memcpy(out + st.param_off, src, st.n_params * 4);
    }
  }
  return MOBIUS_OK;
}

extern "C" int mobius_read_params(mobius_ctx* ctx, float* out, size_t n) {
  int rc = check_ctx(ctx);
  if (rc) return rc;
  drain_updates(ctx);
  MOBIUS_CHECK_ARG(out, "null out");
  for (int ls = 0; ls < (int)ctx->mine.size(); ++ls) {
    const StageDesc& st = ctx->all[ctx->mine[ls]];
    MOBIUS_CHECK_ARG((size_t)(st.param_off + st.n_params) <= n, "output too small");
    if (ctx->dev_tail && ls == 0) {
      if (cudaMemcpy(out + st.param_off, ctx->d_opt, st.n_params * 4, cudaMemcpyDeviceToHost) != cudaSuccess)
        MOBIUS_FAIL(MOBIUS_ECUDA, "read_params: device copy");
    } else {
      std::memcpy(out + st.param_off, ctx->h_master[ls], st.n_params * 4);
    }
  }
  return MOBIUS_OK;
}

extern "C" int mobius_read_trace(mobius_ctx* ctx, int32_t* out, size_t cap, size_t* n) {
  MOBIUS_CHECK_ARG(ctx && out && n, "null argument");
  size_t t = ctx->trace.size() / 3;
  *n = t;
  std::memcpy(out, ctx->trace.data(), std::min(t, cap) * 3 * sizeof(int32_t));
  return MOBIUS_OK;
}

extern "C" int mobius_read_timeline(mobius_ctx* ctx, mobius_timeline_event* out, size_t cap, size_t* n) {
  MOBIUS_CHECK_ARG(ctx && n && (out || cap == 0), "null argument");
  if (ctx->step_count == 0) MOBIUS_FAIL(MOBIUS_ESTATE, "read_timeline: no step has run");
  std::vector<mobius_timeline_event> v;
  auto rel = [&](cudaEvent_t a, double* t) {
    float ms = 0.f;
    if (cudaEventElapsedTime(&ms, ctx->ev_step0, a) != cudaSuccess) return false;
    *t = ms;
    return true;
  };
  auto add = [&](int kind, int stage, cudaEvent_t a, cudaEvent_t b) {
    mobius_timeline_event e;
    e.kind = kind;
    e.stage = stage + 1;
    if (rel(a, &e.t0_ms) && rel(b, &e.t1_ms)) v.push_back(e);
  };
  for (int i = 0; i < ctx->n_parts_last; ++i)
    add(ctx->part_d2d[i] ? MOBIUS_TL_D2D : MOBIUS_TL_H2D, ctx->part_stage[i], ctx->ev_part_a[i], ctx->ev_part_b[i]);
  const int nl = (int)ctx->mine.size();
  for (int xi = 0; xi < 2 * nl; ++xi) {  // exec order: F of local stages ascending, then B descending
    const bool fwd = xi < nl;
    const int ls = fwd ? xi : 2 * nl - 1 - xi;
    add(fwd ? MOBIUS_TL_FWD : MOBIUS_TL_BWD, ctx->mine[ls], ctx->ev_pass_a[xi], ctx->ev_pass_b[xi]);
  }
  for (int ls = nl - 1; ls >= 0; --ls) add(MOBIUS_TL_D2H, ctx->mine[ls], ctx->ev_off_a[ls], ctx->ev_off_b[ls]);
  for (int ls = 0; ls < nl; ++ls)
    if (ctx->ck_off[ls]) {
      add(MOBIUS_TL_CKPT_D2H, ctx->mine[ls], ctx->ev_ck_a[2 * ls], ctx->ev_ck_b[2 * ls]);
      add(MOBIUS_TL_CKPT_H2D, ctx->mine[ls], ctx->ev_ck_a[2 * ls + 1], ctx->ev_ck_b[2 * ls + 1]);
    }
  cudaGetLastError();  // clear a not-ready / unrecorded event status
  *n = v.size();
  if (out) std::memcpy(out, v.data(), std::min(cap, v.size()) * sizeof(mobius_timeline_event));
  return MOBIUS_OK;
}

extern "C" int mobius_stats(mobius_ctx* ctx, mobius_step_stats* out) {
  MOBIUS_CHECK_ARG(ctx && out, "null argument");
  *out = ctx->stats;
  return MOBIUS_OK;
}

extern "C" void mobius_destroy(mobius_ctx* ctx) {
  delete ctx;  // ~mobius_ctx: join the update thread, free HBM / pinned / host state, streams and events
}
