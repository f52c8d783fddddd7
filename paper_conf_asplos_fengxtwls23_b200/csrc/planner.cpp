// mobius_plan: partition MIP (PAPER §3.2, Eq 3-11, Table 2) and
// cross mapping (PAPER §3.3, Eq 12/13).  Host only, exact
// integer arithmetic (int64 ns/bytes, ceil transfer times via __int128,
// exact rational contention via a 192-bit accumulator).
//
// For a fixed partition the MIP optimum is the earliest-start recurrence
// (every constraint is t >= monotone function of earlier t), DESIGN.md
// "Planner".  Readings: #5 physical K, #6 W_h / W_p2p, #7 mem vs xfer,
// #8 prefetch window = stage j-N's window, #13 tie-breaks, #14 arithmetic.
#include <algorithm>
#include <cstring>
#include <dirent.h>
#include <limits.h>
#include <map>
#include <numeric>
#include <stdlib.h>
#include <vector>

#include "common.h"

namespace mobius {

namespace {

struct StageSum {
  int64_t Tf, Tb, Sf, Sb, Xf, Xb, A;
};

thread_local int64_t g_last_plan_nodes = 0;  // branch-and-bound nodes of the last mobius_plan (L' > 20)

int64_t ceil_xfer_ns(int64_t bytes, int64_t bw) {
  if (bw <= 0 || bytes <= 0) return 0;
  __int128 num = (__int128)bytes * 1000000000LL;
  return (int64_t)((num + bw - 1) / bw);
}

std::vector<StageSum> stage_sums(const mobius_layer_profile* L, const int* sizes, int K) {
  std::vector<StageSum> st(K);
  int pos = 0;
  for (int j = 0; j < K; ++j) {
    StageSum s{0, 0, 0, 0, 0, 0, 0};
    for (int i = 0; i < sizes[j]; ++i) {
      const mobius_layer_profile& l = L[pos + i];
      s.Tf += l.t_fwd_ns;
      s.Tb += l.t_bwd_ns;
      s.Sf += l.mem_fwd;
      s.Sb += l.mem_bwd;
      s.Xf += l.xfer_fwd;
      s.Xb += l.xfer_bwd;
    }
    s.A = L[pos + sizes[j] - 1].act_out;
    pos += sizes[j];
    st[j] = s;
  }
  return st;
}

// Returns makespan or -1 if infeasible (Eq 4).  tf/tb optional [K*M].
int64_t cost(const mobius_layer_profile* L, const int* sizes, int K, int N, int64_t G, int M, int64_t Wh,
             int64_t Wp, int64_t* tf_out, int64_t* tb_out, std::vector<int64_t>& tf, std::vector<int64_t>& tb) {
  std::vector<StageSum> S = stage_sums(L, sizes, K);
  for (int j = 0; j < K; ++j)
    if (S[j].Sf > G || S[j].Sb > G) return -1;
  tf.assign((size_t)K * M, 0);
  tb.assign((size_t)K * M, 0);
  auto p2p = [&](int64_t b) -> int64_t { return N == 1 ? 0 : ceil_xfer_ns(b, Wp); };
  auto pre = [&](int64_t X, int64_t Sp, int64_t B, int64_t E) -> int64_t {
    // Eq 5/6/9: P <= min(G - S_p, W*D_p, X); t >= E + (X - P)/W
    int64_t a = E;
    int64_t b = E + ceil_xfer_ns(std::max<int64_t>(0, X - (G - Sp)), Wh);
    int64_t c = B + ceil_xfer_ns(X, Wh);
    return std::max(a, std::max(b, c));
  };
#define TF(j, m) tf[(size_t)(j) * M + (m)]
#define TB(j, m) tb[(size_t)(j) * M + (m)]
  for (int j = 0; j < K; ++j) {
    for (int m = 0; m < M; ++m) {
      int64_t t = 0;
      if (m > 0) t = std::max(t, TF(j, m - 1) + S[j].Tf);                        // Eq 10
      if (j > 0) t = std::max(t, TF(j - 1, m) + S[j - 1].Tf + p2p(S[j - 1].A));  // Eq 8
      if (m == 0 && j >= N) {                                                     // Eq 9
        int p = j - N;
        t = std::max(t, pre(S[j].Xf, S[p].Sf, TF(p, 0), TF(p, M - 1) + S[p].Tf));
      }
      TF(j, m) = t;
    }
  }
  for (int j = K - 1; j >= 0; --j) {
    for (int m = 0; m < M; ++m) {
      int64_t t = 0;
      if (m > 0) t = std::max(t, TB(j, m - 1) + S[j].Tb);
      if (j < K - 1) t = std::max(t, TB(j + 1, m) + S[j + 1].Tb + p2p(S[j].A));
      if (j == K - 1 && m == 0) t = std::max(t, TF(K - 1, M - 1) + S[K - 1].Tf);  // Eq 11
      if (m == 0 && j + N <= K - 1) {
        int p = j + N;
        t = std::max(t, pre(S[j].Xb, S[p].Sb, TB(p, 0), TB(p, M - 1) + S[p].Tb));
      }
      TB(j, m) = t;
    }
  }
  int64_t mk = TB(0, M - 1) + S[0].Tb;  // Eq 3
#undef TF
#undef TB
  if (tf_out) std::memcpy(tf_out, tf.data(), sizeof(int64_t) * K * M);
  if (tb_out) std::memcpy(tb_out, tb.data(), sizeof(int64_t) * K * M);
  return mk;
}

// key (makespan, K, sizes lexicographic) - reading #13
bool better(int64_t mk, const std::vector<int>& sizes, int64_t best_mk, const std::vector<int>& best) {
  if (best.empty()) return true;
  if (mk != best_mk) return mk < best_mk;
  if (sizes.size() != best.size()) return sizes.size() < best.size();
  return sizes < best;
}

// ---------------- exact rational contention ------------------------------
typedef unsigned __int128 u128;

struct U192 {
  uint64_t w[3] = {0, 0, 0};
  void add(u128 v) {
    uint64_t lo = (uint64_t)v, hi = (uint64_t)(v >> 64);
    uint64_t s0 = w[0] + lo;
    uint64_t c0 = s0 < w[0];
    uint64_t s1 = w[1] + hi;
    uint64_t c1 = s1 < w[1];
    uint64_t s1b = s1 + c0;
    c1 |= s1b < s1;
    w[0] = s0;
    w[1] = s1b;
    w[2] += c1;
  }
  bool operator<(const U192& o) const {
    for (int i = 2; i >= 0; --i)
      if (w[i] != o.w[i]) return w[i] < o.w[i];
    return false;
  }
  bool operator==(const U192& o) const { return w[0] == o.w[0] && w[1] == o.w[1] && w[2] == o.w[2]; }
  long double as_ld() const {
    return (long double)w[2] * 18446744073709551616.0L * 18446744073709551616.0L +
           (long double)w[1] * 18446744073709551616.0L + (long double)w[0];
  }
};

u128 gcd128(u128 a, u128 b) {
  while (b) {
    u128 t = a % b;
    a = b;
    b = t;
  }
  return a;
}

struct ContentionModel {
  int K, N;
  u128 D = 1;                       // lcm(1..K-1)
  std::vector<u128> W;              // W[a*N+b], a<b: sum over stage pairs of D/d
  std::vector<int> gsize;           // group size per group id
  bool ok = true;
  ContentionModel(int K_, int N_, const int* group) : K(K_), N(N_) {
    for (int d = 2; d <= K - 1; ++d) {
      u128 g = gcd128(D, (u128)d);
      u128 nd = D / g * d;
      if (nd / d != D / g) {
        ok = false;
        return;
      }
      D = nd;
    }
    W.assign((size_t)N * N, 0);
    for (int i = 0; i < K; ++i)
      for (int j = i + 1; j < K; ++j) {
        int a = i % N, b = j % N;
        if (a == b) continue;  // same GPU: excluded (reading #12)
        if (a > b) std::swap(a, b);
        W[(size_t)a * N + b] += D / (u128)(j - i);
      }
    int mx = 0;
    for (int g = 0; g < N; ++g) mx = std::max(mx, group[g]);
    gsize.assign(mx + 1, 0);
    for (int g = 0; g < N; ++g) gsize[group[g]]++;
  }
  U192 eval(const int* perm, const int* group) const {
    U192 acc;
    for (int a = 0; a < N; ++a)
      for (int b = a + 1; b < N; ++b) {
        int ga = perm[a], gb = perm[b];
        if (group[ga] != group[gb]) continue;
        u128 w = W[(size_t)a * N + b];
        for (int r = 0; r < gsize[group[ga]]; ++r) acc.add(w);
      }
    return acc;
  }
  void output(const U192& v, double* c, int64_t* num, int64_t* den) const {
    if (c) *c = (double)(v.as_ld() / (long double)D);
    int64_t n = 0, d = 0;
    if (v.w[2] == 0) {
      u128 nv = ((u128)v.w[1] << 64) | v.w[0];
      u128 g = gcd128(nv, D);
      if (g == 0) g = 1;
      u128 rn = nv / g, rd = D / g;
      if (rn <= (u128)INT64_MAX && rd <= (u128)INT64_MAX) {
        n = (int64_t)rn;
        d = (int64_t)rd;
      }
    }
    if (num) *num = n;
    if (den) *den = d;
  }
};

int validate_profile(const mobius_layer_profile* layers, int n) {
  MOBIUS_CHECK_ARG(layers != nullptr && n >= 1 && n <= MOBIUS_MAX_LAYERS, "bad layer profile (n=%d)", n);
  for (int i = 0; i < n; ++i) {
    const mobius_layer_profile& l = layers[i];
    MOBIUS_CHECK_ARG(l.t_fwd_ns >= 0 && l.t_bwd_ns >= 0 && l.mem_fwd >= 0 && l.mem_bwd >= 0 && l.xfer_fwd >= 0 &&
                         l.xfer_bwd >= 0 && l.act_out >= 0,
                     "negative profile entry at layer %d", i);
  }
  return MOBIUS_OK;
}

void balanced_sizes(const mobius_layer_profile* L, int n, int K, std::vector<int>& out) {
  // split by cumulative (t_fwd + t_bwd + 1) so stages carry ~equal compute
  std::vector<double> w(n);
  double tot = 0;
  for (int i = 0; i < n; ++i) {
    w[i] = (double)(L[i].t_fwd_ns + L[i].t_bwd_ns) + 1.0;
    tot += w[i];
  }
  out.clear();
  int start = 0;
  double acc = 0;
  for (int j = 0; j < K; ++j) {
    int remaining_stages = K - j;
    int max_end = n - (remaining_stages - 1);
    double target = tot * (j + 1) / K;
    int end = start + 1;
    acc += w[start];
    while (end < max_end && acc + w[end] * 0.5 <= target) {
      acc += w[end];
      ++end;
    }
    if (j == K - 1) {
      while (end < n) acc += w[end++];
    }
    out.push_back(end - start);
    start = end;
  }
}

}  // namespace

int plan_cost_impl(const mobius_layer_profile* layers, int n_layers, const int* sizes, int K, int N, int64_t G, int M,
                   int64_t Wh, int64_t Wp, int64_t* mk, int64_t* tf, int64_t* tb) {
  std::vector<int64_t> a, b;
  int64_t r = cost(layers, sizes, K, N, G, M, Wh, Wp, tf, tb, a, b);
  if (r < 0) MOBIUS_FAIL(MOBIUS_EINFEASIBLE, "partition infeasible under cap %lld", (long long)G);
  *mk = r;
  return MOBIUS_OK;
}

}  // namespace mobius

using namespace mobius;

extern "C" int mobius_plan_cost(const mobius_layer_profile* layers, int n_layers, const int* stage_sizes,
                                int n_stages, int n_gpus, int64_t G, int M, int64_t Wh, int64_t Wp,
                                int64_t* makespan_ns, int64_t* tf, int64_t* tb) {
  int rc = validate_profile(layers, n_layers);
  if (rc) return rc;
  MOBIUS_CHECK_ARG(stage_sizes && n_stages >= 1 && n_gpus >= 1 && M >= 1 && makespan_ns, "bad arguments");
  int tot = 0;
  for (int j = 0; j < n_stages; ++j) {
    MOBIUS_CHECK_ARG(stage_sizes[j] >= 1, "empty stage %d", j);
    tot += stage_sizes[j];
  }
  MOBIUS_CHECK_ARG(tot == n_layers, "stage sizes sum %d != %d layers", tot, n_layers);
  return plan_cost_impl(layers, n_layers, stage_sizes, n_stages, n_gpus, G, M, Wh, Wp, makespan_ns, tf, tb);
}

extern "C" int mobius_mapping_contention(int K, int N, const int* group, const int* perm, double* c, int64_t* num,
                                         int64_t* den) {
  MOBIUS_CHECK_ARG(K >= 1 && N >= 1 && N <= MOBIUS_MAX_GPUS && group && perm, "bad arguments");
  ContentionModel cm(K, N, group);
  MOBIUS_CHECK_ARG(cm.ok, "too many stages (%d) for exact contention", K);
  cm.output(cm.eval(perm, group), c, num, den);
  return MOBIUS_OK;
}

extern "C" int mobius_cross_map(int K, int N, const int* group, int* perm_out, double* c, int64_t* num,
                                int64_t* den) {
  MOBIUS_CHECK_ARG(K >= 1 && N >= 1 && N <= 10 && group && perm_out, "bad arguments (N=%d)", N);
  ContentionModel cm(K, N, group);
  MOBIUS_CHECK_ARG(cm.ok, "too many stages (%d) for exact contention", K);
  std::vector<int> perm(N), best;
  std::iota(perm.begin(), perm.end(), 0);
  U192 bv;
  do {  // lexicographic order: first strict minimum = tie-break of reading #13
    U192 v = cm.eval(perm.data(), group);
    if (best.empty() || v < bv) {
      bv = v;
      best = perm;
    }
  } while (std::next_permutation(perm.begin(), perm.end()));
  std::copy(best.begin(), best.end(), perm_out);
  cm.output(bv, c, num, den);
  return MOBIUS_OK;
}

// Exact partition search for L' > 20 (branch and bound over stage
// boundaries, left to right).  For a prefix ending with stage j (first layer
// a_j) the forward start times t^f of the prefix are final (Eq 8-10 only look
// at earlier stages), and the dependency chain F_{j,M} -> ... -> F_{K,M} ->
// B_{K,1} (Eq 11) -> ... -> B_{1,1} -> ... -> B_{1,M} (Eq 8 / 10) bounds the
// makespan of every completion from below:
//   LB = t^f_{j,M} + sum_{i >= a_j} t_f(i) + sum_i t_b(i) + (M - 1) T^b_1
// (transfer terms >= 0 dropped; the sums are partition independent).  Ties
// of the key (makespan, K, sizes) prune through the fewest stages any
// completion needs (greedy packing from a_j) and the lexicographic order of
// the prefix.  The local-search result seeds the incumbent; a node budget
// (MOBIUS_PLAN_BNB_NODES, default 1M at N = 1, 200k otherwise) bounds the work - when it is hit the
// search is not a certificate and the incumbent is returned.
struct BnB {
  const mobius_layer_profile* L;
  int n, N, M;
  int64_t G, Wh, Wp;
  std::vector<int64_t> sf_suffix;   // sum t_f over layers >= i
  int64_t sb_all = 0;
  std::vector<int> min_stages;      // fewest stages covering layers >= i
  std::vector<int> sizes;           // current prefix
  std::vector<StageSum> st;         // prefix stage sums
  std::vector<std::vector<int64_t>> tf;  // prefix forward start rows
  std::vector<int> best;
  int64_t best_mk = -1;
  int64_t nodes = 0, node_limit = 0;
  bool aborted = false;
  std::vector<int64_t> wa, wb;

  int64_t p2p(int64_t b) const { return N == 1 ? 0 : ceil_xfer_ns(b, Wp); }

  void init() {
    sf_suffix.assign(n + 1, 0);
    for (int i = n - 1; i >= 0; --i) sf_suffix[i] = sf_suffix[i + 1] + L[i].t_fwd_ns;
    for (int i = 0; i < n; ++i) sb_all += L[i].t_bwd_ns;
    min_stages.assign(n + 1, 0);
    for (int i = n - 1; i >= 0; --i) {  // greedy packing from i is the fewest contiguous stages
      int cnt = 0, pos = i;
      while (pos < n) {
        int64_t a = 0, b = 0;
        int q = pos;
        while (q < n && a + L[q].mem_fwd <= G && b + L[q].mem_bwd <= G) {
          a += L[q].mem_fwd;
          b += L[q].mem_bwd;
          ++q;
        }
        if (q == pos) {
          cnt = INT_MAX / 2;
          break;
        }
        ++cnt;
        pos = q;
      }
      min_stages[i] = cnt;
    }
  }
  // forward row of stage j = sizes.size()-1 (its sums in st.back())
  void push_row() {
    const int j = (int)st.size() - 1;
    std::vector<int64_t> row(M, 0);
    for (int m = 0; m < M; ++m) {
      int64_t t = 0;
      if (m > 0) t = std::max(t, row[m - 1] + st[j].Tf);
      if (j > 0) t = std::max(t, tf[j - 1][m] + st[j - 1].Tf + p2p(st[j - 1].A));
      if (m == 0 && j >= N) {
        const int q = j - N;
        const int64_t B = tf[q][0], E = tf[q][M - 1] + st[q].Tf;
        t = std::max(t, std::max(E, std::max(E + ceil_xfer_ns(std::max<int64_t>(0, st[j].Xf - (G - st[q].Sf)), Wh),
                                             B + ceil_xfer_ns(st[j].Xf, Wh))));
      }
      row[m] = t;
    }
    tf.push_back(row);
  }
  // false: no completion of the prefix can beat the incumbent's key
  bool may_improve(int pos) const {
    if (best_mk < 0) return true;
    const int j = (int)st.size() - 1;
    int64_t lb = tf[j][M - 1] + sf_suffix[pos - sizes.back()] + sb_all + (int64_t)(M - 1) * st[0].Tb;
    // one GPU runs everything serially: after F_{j,M} it still runs M
    // forwards of every later layer and M backwards of every layer
    if (N == 1) lb = std::max(lb, tf[j][M - 1] + st[j].Tf + (int64_t)M * (sf_suffix[pos] + sb_all));
    if (lb > best_mk) return false;
    if (lb < best_mk) return true;
    const int k_lb = (int)sizes.size() + (pos < n ? min_stages[pos] : 0);
    if (k_lb > (int)best.size()) return false;
    if (k_lb < (int)best.size()) return true;
    // same K possible: the completion's sizes start with the prefix
    for (size_t i = 0; i < sizes.size() && i < best.size(); ++i) {
      if (sizes[i] != best[i]) return sizes[i] < best[i];
    }
    return true;
  }
  void dfs(int pos) {
    if (aborted) return;
    if (++nodes > node_limit) {
      aborted = true;
      return;
    }
    if (pos == n) {
      const int64_t mk = cost(L, sizes.data(), (int)sizes.size(), N, G, M, Wh, Wp, nullptr, nullptr, wa, wb);
      if (mk >= 0 && better(mk, sizes, best_mk, best)) {
        best_mk = mk;
        best = sizes;
      }
      return;
    }
    StageSum s{0, 0, 0, 0, 0, 0, 0};
    for (int len = 1; pos + len <= n; ++len) {
      const mobius_layer_profile& l = L[pos + len - 1];
      s.Tf += l.t_fwd_ns;
      s.Tb += l.t_bwd_ns;
      s.Sf += l.mem_fwd;
      s.Sb += l.mem_bwd;
      s.Xf += l.xfer_fwd;
      s.Xb += l.xfer_bwd;
      s.A = l.act_out;
      if (s.Sf > G || s.Sb > G) break;  // longer stages only grow (Eq 4)
      sizes.push_back(len);
      st.push_back(s);
      push_row();
      if (may_improve(pos + len)) dfs(pos + len);
      tf.pop_back();
      st.pop_back();
      sizes.pop_back();
      if (aborted) return;
    }
  }
};

// brute force over all 2^(L'-1) compositions up to this many profile layers
// (MOBIUS_PLAN_EXHAUSTIVE_MAX, default 20, at most 26: tests compare it with
// the branch and bound just above 20)
static int exhaustive_limit() {
  int v = 20;
  if (const char* e = getenv("MOBIUS_PLAN_EXHAUSTIVE_MAX")) v = std::min(26, std::max(1, atoi(e)));
  return v;
}

static int plan_impl(const mobius_layer_profile* layers, int n_layers, int N, int64_t G, int M,
                     const mobius_topology* topo_in, int algo, mobius_plan_t* out) {
  int rc = validate_profile(layers, n_layers);
  if (rc) return rc;
  MOBIUS_CHECK_ARG(out && N >= 1 && N <= MOBIUS_MAX_GPUS && M >= 1 && G > 0, "bad arguments");
  mobius_topology topo;
  if (topo_in) {
    topo = *topo_in;
  } else {
    rc = mobius_discover_topology(&topo);
    if (rc) return rc;
  }
  MOBIUS_CHECK_ARG(topo.n_gpus >= N, "topology has %d GPUs < %d", topo.n_gpus, N);
  for (int i = 0; i < n_layers; ++i)
    if (layers[i].mem_fwd > G || layers[i].mem_bwd > G)
      MOBIUS_FAIL(MOBIUS_EINFEASIBLE, "layer %d needs %lld bytes > cap %lld", i,
                  (long long)std::max(layers[i].mem_fwd, layers[i].mem_bwd), (long long)G);
  const int64_t Wh = topo.host_bw_Bps, Wp = topo.p2p_bw_Bps;
  g_last_plan_nodes = 0;

  std::vector<int> best;
  int64_t best_mk = -1;
  std::vector<int64_t> a, b;
  int exhaustive = 0;
  if (algo == MOBIUS_PARTITION_MAX_STAGE || algo == MOBIUS_PARTITION_MIN_STAGE) {
    // Fig 9 baselines: as many layers per stage as memory
    // allows (greedy, front to back), or one layer per stage
    if (algo == MOBIUS_PARTITION_MIN_STAGE) {
      best.assign(n_layers, 1);
    } else {
      int cur = 0;
      int64_t sf = 0, sb = 0;
      for (int i = 0; i < n_layers; ++i) {
        if (cur && (sf + layers[i].mem_fwd > G || sb + layers[i].mem_bwd > G)) {
          best.push_back(cur);
          cur = 0;
          sf = sb = 0;
        }
        ++cur;
        sf += layers[i].mem_fwd;
        sb += layers[i].mem_bwd;
      }
      best.push_back(cur);
    }
    best_mk = cost(layers, best.data(), (int)best.size(), N, G, M, Wh, Wp, nullptr, nullptr, a, b);
    if (best_mk < 0) best.clear();
  } else if (n_layers <= exhaustive_limit()) {
    exhaustive = 1;
    std::vector<int> sizes;
    sizes.reserve(n_layers);
    for (uint32_t cuts = 0; cuts < (1u << (n_layers - 1)); ++cuts) {
      sizes.clear();
      int run = 1;
      for (int bit = 0; bit < n_layers - 1; ++bit) {
        if (cuts >> bit & 1u) {
          sizes.push_back(run);
          run = 1;
        } else {
          ++run;
        }
      }
      sizes.push_back(run);
      int64_t mk = cost(layers, sizes.data(), (int)sizes.size(), N, G, M, Wh, Wp, nullptr, nullptr, a, b);
      if (mk < 0) continue;
      if (better(mk, sizes, best_mk, best)) {
        best_mk = mk;
        best = sizes;
      }
    }
  } else {
    // balanced start per K, then first-improvement boundary moves (+-1)
    std::vector<int> sizes;
    for (int K = 1; K <= n_layers; ++K) {
      balanced_sizes(layers, n_layers, K, sizes);
      int64_t mk = cost(layers, sizes.data(), K, N, G, M, Wh, Wp, nullptr, nullptr, a, b);
      bool improved = true;
      int iters = 0;
      while (improved && iters++ < 4 * n_layers) {
        improved = false;
        for (int j = 0; j + 1 < K && !improved; ++j) {
          for (int dir = -1; dir <= 1 && !improved; dir += 2) {
            std::vector<int> t = sizes;
            t[j] += dir;
            t[j + 1] -= dir;
            if (t[j] < 1 || t[j + 1] < 1) continue;
            int64_t m2 = cost(layers, t.data(), K, N, G, M, Wh, Wp, nullptr, nullptr, a, b);
            if (m2 < 0) continue;
            if (mk < 0 || better(m2, t, mk, sizes)) {
              sizes = t;
              mk = m2;
              improved = true;
            }
          }
        }
      }
      if (mk >= 0 && better(mk, sizes, best_mk, best)) {
        best_mk = mk;
        best = sizes;
      }
    }
    // certify (or improve) the local-search result by branch and bound
    BnB bb;
    bb.L = layers;
    bb.n = n_layers;
    bb.N = N;
    bb.M = M;
    bb.G = G;
    bb.Wh = Wh;
    bb.Wp = Wp;
    bb.node_limit = N == 1 ? 1000000 : 200000;  // the N > 1 bounds are weaker: best found
    if (const char* e = getenv("MOBIUS_PLAN_BNB_NODES")) bb.node_limit = atoll(e);
    bb.best = best;
    bb.best_mk = best_mk;
    bb.init();
    if (bb.node_limit > 0) bb.dfs(0);
    if (!bb.best.empty()) {
      best = bb.best;
      best_mk = bb.best_mk;
    }
    exhaustive = (!bb.aborted && bb.node_limit > 0) ? 1 : 0;
    g_last_plan_nodes = bb.nodes;
  }
  if (best.empty()) MOBIUS_FAIL(MOBIUS_EINFEASIBLE, "no feasible partition under cap %lld", (long long)G);

  std::memset(out, 0, sizeof(*out));
  int K = (int)best.size();
  MOBIUS_CHECK_ARG(K <= MOBIUS_MAX_LAYERS, "too many stages");
  out->n_stages = K;
  out->n_gpus = N;
  out->n_microbatches = M;
  out->n_layers = n_layers;
  out->hbm_cap_bytes = G;
  out->makespan_ns = best_mk;
  out->exhaustive = exhaustive;
  out->stage_first_layer[0] = 0;
  for (int j = 0; j < K; ++j) out->stage_first_layer[j + 1] = out->stage_first_layer[j] + best[j];
  int perm[MOBIUS_MAX_GPUS];
  if (N <= 10) {
    rc = mobius_cross_map(K, N, topo.group, perm, &out->contention, &out->contention_num, &out->contention_den);
    if (rc) return rc;
  } else {
    for (int g = 0; g < N; ++g) perm[g] = g;
    rc = mobius_mapping_contention(K, N, topo.group, perm, &out->contention, &out->contention_num,
                                   &out->contention_den);
    if (rc) return rc;
  }
  for (int g = 0; g < N; ++g) out->gpu_perm[g] = perm[g];
  for (int j = 0; j < K; ++j) out->stage_gpu[j] = perm[j % N];
  // byte accounting (O-10, reading #11: 2K - N loads)
  std::vector<StageSum> S = stage_sums(layers, best.data(), K);
  for (int j = 0; j < K; ++j) {
    int g = out->stage_gpu[j];
    out->h2d_bytes[g] += S[j].Xf;
    if (j + N <= K - 1) out->h2d_bytes[g] += S[j].Xb;
    out->d2h_bytes[g] += S[j].Xf;  // gradients in the transfer precision
    if (N > 1 && j < K - 1) {
      out->p2p_bytes[g] += (int64_t)M * S[j].A;
      out->p2p_bytes[out->stage_gpu[j + 1]] += (int64_t)M * S[j].A;
    }
  }
  return MOBIUS_OK;
}

// ---------------------------------------------------------------------------
// topology discovery: group GPUs by PCIe root complex ("pci<domain>:<bus>"
// sysfs ancestor), P:L836-846 / reading #12.
// ---------------------------------------------------------------------------
#include <cuda_runtime.h>

extern "C" int mobius_discover_topology(mobius_topology* out) {
  MOBIUS_CHECK_ARG(out, "null out");
  std::memset(out, 0, sizeof(*out));
  int n = 0;
  cudaError_t e = cudaGetDeviceCount(&n);
  if (e != cudaSuccess || n <= 0) MOBIUS_FAIL(MOBIUS_ETOPO, "no CUDA devices (%s)", cudaGetErrorString(e));
  n = std::min(n, MOBIUS_MAX_GPUS);
  out->n_gpus = n;
  std::map<std::string, int> ids;
  for (int d = 0; d < n; ++d) {
    char bus[64] = {0};
    std::string root = "unknown";
    if (cudaDeviceGetPCIBusId(bus, sizeof(bus), d) == cudaSuccess) {
      for (char* p = bus; *p; ++p) *p = (char)tolower(*p);
      std::string path = std::string("/sys/bus/pci/devices/") + bus;
      char real[PATH_MAX];
      if (realpath(path.c_str(), real)) {
        // /sys/devices/pci0000:15/0000:15:01.0/... -> "pci0000:15"
        std::string r(real);
        size_t p0 = r.find("/pci");
        if (p0 != std::string::npos) {
          size_t p1 = r.find('/', p0 + 1);
          root = r.substr(p0 + 1, p1 == std::string::npos ? std::string::npos : p1 - p0 - 1);
        }
      }
    }
    auto it = ids.find(root);
    if (it == ids.end()) it = ids.emplace(root, (int)ids.size()).first;
    out->group[d] = it->second;
  }
  return MOBIUS_OK;
}

extern "C" int64_t mobius_plan_search_nodes(void) { return g_last_plan_nodes; }

extern "C" int mobius_plan(const mobius_layer_profile* layers, int n_layers, int N, int64_t G, int M,
                           const mobius_topology* topo_in, mobius_plan_t* out) {
  return plan_impl(layers, n_layers, N, G, M, topo_in, MOBIUS_PARTITION_MIP, out);
}

extern "C" int mobius_plan_partition(const mobius_layer_profile* layers, int n_layers, int N, int64_t G, int M,
                                     const mobius_topology* topo_in, int algo, mobius_plan_t* out) {
  MOBIUS_CHECK_ARG(algo == MOBIUS_PARTITION_MIP || algo == MOBIUS_PARTITION_MAX_STAGE ||
                       algo == MOBIUS_PARTITION_MIN_STAGE,
                   "unknown partition algorithm %d", algo);
  return plan_impl(layers, n_layers, N, G, M, topo_in, algo, out);
}

// ---------------------------------------------------------------------------
// measured contention groups: the "root
// complex" that matters is the level at which concurrent pinned H2D copies
// slow each other down; on B200 boxes the PCIe switch / socket layout is not
// visible from sysfs alone.
// ---------------------------------------------------------------------------
extern "C" int mobius_topology_from_bw(int n, const double* solo, const double* pair, double threshold,
                                       mobius_topology* out) {
  MOBIUS_CHECK_ARG(n >= 1 && n <= MOBIUS_MAX_GPUS && solo && (pair || n == 1) && out && threshold > 0 &&
                       threshold <= 1,
                   "bad arguments");
  std::vector<int> parent(n);
  std::iota(parent.begin(), parent.end(), 0);
  auto find = [&](int x) {
    while (parent[x] != x) x = parent[x] = parent[parent[x]];
    return x;
  };
  for (int i = 0; i < n; ++i)
    for (int j = i + 1; j < n; ++j) {
      MOBIUS_CHECK_ARG(solo[i] > 0 && solo[j] > 0, "solo bandwidth must be positive");
      const double ri = pair[i * n + j] / solo[i], rj = pair[j * n + i] / solo[j];
      if (std::min(ri, rj) < threshold) parent[find(i)] = find(j);
    }
  std::memset(out, 0, sizeof(*out));
  out->n_gpus = n;
  std::map<int, int> ids;  // group ids numbered by first member
  for (int i = 0; i < n; ++i) {
    const int r = find(i);
    auto it = ids.find(r);
    if (it == ids.end()) it = ids.emplace(r, (int)ids.size()).first;
    out->group[i] = it->second;
  }
  std::vector<double> s(solo, solo + n);
  std::sort(s.begin(), s.end());
  out->host_bw_Bps = (int64_t)(s[n / 2] * 1e9);
  return MOBIUS_OK;
}

extern "C" int mobius_probe_topology(int64_t bytes, double threshold, mobius_topology* out, double* solo_out,
                                     double* pair_out) {
  MOBIUS_CHECK_ARG(out && bytes >= (1 << 20), "bad arguments");
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess || n <= 0) MOBIUS_FAIL(MOBIUS_ETOPO, "no CUDA devices");
  n = std::min(n, MOBIUS_MAX_GPUS);
  int cur = 0;
  cudaGetDevice(&cur);
  std::vector<void*> h(n, nullptr), d(n, nullptr);
  std::vector<cudaStream_t> st(n, nullptr);
  std::vector<cudaEvent_t> ea(n, nullptr), eb(n, nullptr);
  int rc = MOBIUS_OK;
  auto cleanup = [&]() {
    for (int i = 0; i < n; ++i) {
      cudaSetDevice(i);
      if (st[i]) cudaStreamSynchronize(st[i]);
      if (h[i]) cudaFreeHost(h[i]);
      if (d[i]) cudaFree(d[i]);
      if (st[i]) cudaStreamDestroy(st[i]);
      if (ea[i]) cudaEventDestroy(ea[i]);
      if (eb[i]) cudaEventDestroy(eb[i]);
    }
    cudaSetDevice(cur);
  };
  for (int i = 0; i < n && !rc; ++i) {
    if (cudaSetDevice(i) != cudaSuccess || cudaMalloc(&d[i], bytes) != cudaSuccess ||
        cudaHostAlloc(&h[i], bytes, cudaHostAllocPortable) != cudaSuccess ||
        cudaStreamCreateWithFlags(&st[i], cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreate(&ea[i]) != cudaSuccess || cudaEventCreate(&eb[i]) != cudaSuccess)
      rc = MOBIUS_ENOMEM;
    else
      std::memset(h[i], 1, bytes);
  }
  if (rc) {
    cleanup();
    MOBIUS_FAIL(rc, "probe_topology: allocation");
  }
  const int reps = 3;
  // run the copies of GPUs in `set` concurrently, return per-GPU GB/s
  auto measure = [&](const std::vector<int>& set, std::vector<double>& gbps) -> int {
    for (int pass = 0; pass < 2; ++pass) {  // pass 0 warms up
      for (int i : set) {
        cudaSetDevice(i);
        cudaEventRecord(ea[i], st[i]);
      }
      for (int k = 0; k < reps; ++k)
        for (int i : set) {
          cudaSetDevice(i);
          cudaMemcpyAsync(d[i], h[i], bytes, cudaMemcpyHostToDevice, st[i]);
        }
      for (int i : set) {
        cudaSetDevice(i);
        cudaEventRecord(eb[i], st[i]);
      }
      for (int i : set) {
        cudaSetDevice(i);
        if (cudaStreamSynchronize(st[i]) != cudaSuccess) return MOBIUS_ECUDA;
      }
    }
    gbps.assign(n, 0.0);
    for (int i : set) {
      float ms = 0.f;
      cudaEventElapsedTime(&ms, ea[i], eb[i]);
      gbps[i] = ms > 0 ? reps * (double)bytes / (ms * 1e-3) / 1e9 : 0.0;
    }
    return MOBIUS_OK;
  };
  std::vector<double> solo(n), pair((size_t)n * n, 0.0), g;
  for (int i = 0; i < n && !rc; ++i) {
    rc = measure({i}, g);
    solo[i] = g[i];
  }
  for (int i = 0; i < n && !rc; ++i)
    for (int j = i + 1; j < n && !rc; ++j) {
      rc = measure({i, j}, g);
      pair[(size_t)i * n + j] = g[i];
      pair[(size_t)j * n + i] = g[j];
    }
  int64_t p2p = 0;
  if (!rc && n >= 2) {  // GPU0 -> GPU1 over NVLink (peer copy)
    int can = 0;
    cudaDeviceCanAccessPeer(&can, 1, 0);
    if (can) {
      cudaSetDevice(1);
      cudaDeviceEnablePeerAccess(0, 0);
      cudaGetLastError();
      cudaSetDevice(0);
      cudaEventRecord(ea[0], st[0]);
      for (int k = 0; k < reps; ++k) cudaMemcpyPeerAsync(d[1], 1, d[0], 0, bytes, st[0]);
      cudaEventRecord(eb[0], st[0]);
      cudaStreamSynchronize(st[0]);
      float ms = 0.f;
      cudaEventElapsedTime(&ms, ea[0], eb[0]);
      if (ms > 0) p2p = (int64_t)(reps * (double)bytes / (ms * 1e-3));
    }
  }
  cleanup();
  if (rc) MOBIUS_FAIL(rc, "probe_topology: copy failed");
  rc = mobius_topology_from_bw(n, solo.data(), pair.data(), threshold, out);
  if (rc) return rc;
  out->p2p_bw_Bps = p2p;
  if (solo_out) std::copy(solo.begin(), solo.end(), solo_out);
  if (pair_out) std::copy(pair.begin(), pair.end(), pair_out);
  return MOBIUS_OK;
}
