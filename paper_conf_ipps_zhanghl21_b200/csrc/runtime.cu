// Device runtime: the compiled program of a bound graph, the executor and the profiler.
//
//  * Program  — one "compiled subgraph" per IR node ("going through the DL
//    compilation pipeline"): the node's sm_100a kernels, prepared weights (BN folded, RNN gates
//    block-interleaved), TMA descriptors and its library-owned output buffer.
//  * Executor — PAPER.md:82 (§IV-D) spawns two busy-looping processes fed by shared-memory
//    queues; on a B200 the equivalent is ONE CUDA graph per schedule: every subgraph's kernels are
//    captured on its slot's stream in schedule order, cross-slot dependencies become event edges
//    (the sync queue), and a replay is a single cudaGraphLaunch on the home stream.
//  * Profiler — PAPER.md:80 (§IV-B) / :87 (500 runs): each subgraph is captured alone and timed
//    with CUDA events (samples of R replays; lower median, int64 ns).
#include <chrono>
#include <algorithm>
#include <cstring>
#include <functional>

#include "common.h"
#include "kernels/kernels.h"

namespace duet {

// fp32 contractions on the tensor cores (3xTF32, gemm_tf32.cu); DUET_TF32=0 keeps the CUDA-core
// kernels (comparisons)
static bool tf32_on() {
  static const bool on = !(getenv("DUET_TF32") && atoi(getenv("DUET_TF32")) == 0);
  return on;
}

// ------------------------------------------------------------------------------------------------
// Program
// ------------------------------------------------------------------------------------------------
using Ptrs = std::vector<void*>;

struct Op {
  std::function<void(const Ptrs&, cudaStream_t)> launch;
  int n_kernels = 0;
};

struct Program {
  const Graph* g = nullptr;
  int device = 0;
  std::vector<void*> buf;                  // per node: library output buffer (inputs: staging)
  std::vector<Op> ops;                     // per node
  std::vector<void*> allocs;               // device memory to free
  std::map<int, std::pair<int, int>> fuse_res;  // conv node -> (residual node, add node it writes)
  std::set<int> fused_adds;
  ~Program() {
    int prev = 0;
    cudaGetDevice(&prev);
    cudaSetDevice(device);
    for (void* p : allocs) cudaFree(p);
    cudaSetDevice(prev);
  }
  void* alloc(int64_t bytes) {
    void* p = nullptr;
    if (bytes <= 0) bytes = 16;
    cudaError_t e = cudaMalloc(&p, (size_t)((bytes + 255) / 256 * 256));
    if (e != cudaSuccess) {
      cudaGetLastError();
      fail(e == cudaErrorMemoryAllocation ? DUET_ENOMEM : DUET_ECUDA,
           std::string("cudaMalloc(") + std::to_string(bytes) + "): " + cudaGetErrorString(e));
    }
    allocs.push_back(p);
    return p;
  }
  void* param(const std::string& name) const {
    auto it = g->bound.find(name);
    if (it == g->bound.end()) fail(DUET_EUNBOUND, "parameter @" + name + " is not bound");
    return it->second.data;
  }
};

void destroy_program(Program* p) { delete p; }

namespace {

struct DeviceGuard {
  int prev = 0;
  explicit DeviceGuard(int d) {
    CK(cudaGetDevice(&prev));
    if (prev != d) CK(cudaSetDevice(d));
  }
  ~DeviceGuard() { cudaSetDevice(prev); }
};

int act_code(const std::string& a) {
  if (a == "none") return ACT_NONE;
  if (a == "relu") return ACT_RELU;
  if (a == "sigmoid") return ACT_SIGMOID;
  if (a == "tanh") return ACT_TANH;
  if (a == "gelu") return ACT_GELU;
  fail(DUET_EPARSE, "unknown activation '" + a + "'");
}

void need_dtype(const Node& n, int have, int want, const std::string& what) {
  if (have != want)
    fail(DUET_EDTYPE, "%" + n.name + ": " + what + " is " + dtype_name(have) + ", expected " + dtype_name(want));
}

bool is_float(int d) { return d == kF32 || d == kBF16; }

// combined RNN input bias in the (possibly reordered) column layout:
//   LSTM: b_ih + b_hh for all gates; GRU: b_ih + b_hh for r,z; b_ih only for n (b_hn is applied
//   inside r*(...), PyTorch convention).
__global__ void rnn_bias_kernel(const float* bih, const float* bhh, const int32_t* old_of_new, float* out, int n_new,
                                int H, int is_gru) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n_new) return;
  int o = old_of_new[i];
  if (o < 0) {
    out[i] = 0.0f;
    return;
  }
  float b = bih[o];
  if (!(is_gru && o >= 2 * H)) b += bhh[o];
  out[i] = b;
}

int rnn_step_bn(int kind, int B, int H, int sms) {
  // tile width for the recurrent step: LSTM u in {16,32,64} (BN = 4u), GRU u in {16,32,64} (BN = 3u)
  (void)kind;
  const int G = 4;  // fused step: 4 gate blocks for LSTM and GRU
  const int mt = (B + 127) / 128;
  int best = 0;
  for (int u : {64, 32, 16}) {
    int tiles = mt * ((H + u - 1) / u);
    best = G * u;
    if (tiles >= sms / 2) return G * u;  // enough CTAs: keep the wider tile
  }
  return best;  // u = 16: most CTAs
}

void build_op(Program& P, const Node& n, Op& op) {
  const Graph& g = *P.g;
  auto argn = [&](int i) -> const Node& { return g.nodes[n.arg_nodes.at(i)]; };
  auto pdecl = [&](int i) -> const ParamDecl& { return g.params.at(n.params.at(i)); };
  auto nargs = [&](size_t k, size_t p) {
    if (n.arg_nodes.size() != k || n.params.size() != p)
      fail(DUET_EPARSE, "%" + n.name + " = " + n.op + ": wrong number of arguments");
  };
  const int me = n.id;
  const int sms = num_sms(P.device);

  if (n.op == "input") return;
  if (n.op == "opaque") fail(DUET_EUNSUPPORTED, "%" + n.name + ": opaque nodes have no kernel");

  if (n.op == "hash_mod") {
    nargs(1, 0);
    need_dtype(n, argn(0).dtype, kI64, "input");
    need_dtype(n, n.dtype, kI32, "output");
    const int in = n.arg_nodes[0];
    const int64_t V = n.attr_int("V", 0), cnt = n.numel();
    if (V <= 0 || V > INT32_MAX) fail(DUET_EINVAL, "%" + n.name + ": V out of range");
    op.launch = [=](const Ptrs& T, cudaStream_t st) { hash_mod((const int64_t*)T[in], (int32_t*)T[me], cnt, V, st); };
    op.n_kernels = 1;
  } else if (n.op == "gather_sum") {
    nargs(1, 2);
    need_dtype(n, argn(0).dtype, kI32, "ids");
    need_dtype(n, n.dtype, kF32, "output");
    const auto& t = pdecl(0);
    if (t.shape.size() != 2 || argn(0).shape.size() != 2 || t.shape[0] != argn(0).shape[1])
      fail(DUET_ESHAPE, "%" + n.name + ": table must be [F, R] with F = ids.shape[1]");
    const int in = n.arg_nodes[0], B = (int)argn(0).shape[0], F = (int)argn(0).shape[1];
    const int64_t R = t.shape[1];
    const int tb = t.dtype == kBF16;
    void* T0 = P.param(n.params[0]);
    const float* b = (const float*)P.param(n.params[1]);
    op.launch = [=](const Ptrs& T, cudaStream_t st) {
      gather_sum((const int32_t*)T[in], T0, tb, b, (float*)T[me], B, F, R, st);
    };
    op.n_kernels = 1;
  } else if (n.op == "gather_concat") {
    nargs(1, 1);
    need_dtype(n, argn(0).dtype, kI32, "ids");
    const auto& e = pdecl(0);
    need_dtype(n, n.dtype, e.dtype, "output");
    if (e.shape.size() != 3 || e.shape[0] != argn(0).shape[1])
      fail(DUET_ESHAPE, "%" + n.name + ": table must be [F, R, D]");
    const int in = n.arg_nodes[0], B = (int)argn(0).shape[0], F = (int)argn(0).shape[1], D = (int)e.shape[2];
    const int64_t R = e.shape[1];
    const int es = dtype_bytes(e.dtype);
    void* E = P.param(n.params[0]);
    op.launch = [=](const Ptrs& T, cudaStream_t st) {
      gather_concat((const int32_t*)T[in], E, es, T[me], B, F, R, D, st);
    };
    op.n_kernels = 1;
  } else if (n.op == "embed_seq") {
    nargs(1, 1);
    need_dtype(n, argn(0).dtype, kI32, "tokens");
    const auto& e = pdecl(0);
    need_dtype(n, n.dtype, e.dtype, "output");
    const int in = n.arg_nodes[0], B = (int)argn(0).shape[0], S = (int)argn(0).shape[1], D = (int)e.shape[1];
    const int64_t V = e.shape[0];
    const int es = dtype_bytes(e.dtype);
    void* E = P.param(n.params[0]);
    op.launch = [=](const Ptrs& T, cudaStream_t st) {
      embed_seq((const int32_t*)T[in], E, es, T[me], B, S, V, D, st);
    };
    op.n_kernels = 1;
  } else if (n.op == "linear") {
    nargs(1, 2);
    const Node& x = argn(0);
    const auto& w = pdecl(0);
    if (w.shape.size() != 2 || x.shape.size() != 2 || w.shape[1] != x.shape[1] || n.shape[1] != w.shape[0])
      fail(DUET_ESHAPE, "%" + n.name + ": linear shapes");
    const int in = n.arg_nodes[0], M = (int)x.shape[0], K = (int)x.shape[1], N = (int)w.shape[0];
    const int act = act_code(n.attr_str("act", "none"));
    void* W = P.param(n.params[0]);
    const float* b = (const float*)P.param(n.params[1]);
    const int xb = x.dtype == kBF16, wb = w.dtype == kBF16, yb = n.dtype == kBF16;
    const char* gemm_env = getenv("DUET_GEMM");  // 1 = force the single-CTA tile (comparisons)
    const bool pair = !(gemm_env && atoi(gemm_env) == 1) && M > 128;
    if (xb && wb && K % 8 == 0 && N >= 16 && pair) {
      const char* bn_env = getenv("DUET_GEMM_BN");
      const int bn = bn_env ? atoi(bn_env) : tc2_pick_bn(M, N, K, sms);
      const char* dbg_env = getenv("DUET_GEMM_DBG");
      const int dbg2 = dbg_env ? atoi(dbg_env) : 0;
      CUtensorMap tw = make_tmap_bf16_2d(W, N, K, bn / 2);
      op.launch = [=](const Ptrs& T, cudaStream_t st) {
        CUtensorMap ta = make_tmap_bf16_2d(T[in], M, K, 128);
        TcEpilogue ep;
        ep.bias = b;
        ep.out = T[me];
        ep.ldo = N;
        ep.act = act;
        ep.dbg = dbg2;
        gemm_tc2_maps(ta, tw, M, N, K, bn, ep, yb, st);
      };
    } else if (xb && wb && K % 8 == 0 && N >= 16) {
      const char* dbg_env = getenv("DUET_GEMM_DBG");
      const int dbg = dbg_env ? atoi(dbg_env) : 0;
      const char* bn_env = getenv("DUET_GEMM_BN");
      int bn = bn_env ? atoi(bn_env) : tc_pick_bn(M, N, sms);
      // skinny GEMM (MT-DNN at batch 1: M = 128, K up to 3072): 64-wide tiles split along K
      int splits = tc_splitk(M, N, K, bn_env ? bn : 64, sms);
      if (splits > 1 && !bn_env) bn = 64;
      float* ws = splits > 1 ? (float*)P.alloc((int64_t)splits * M * N * 4) : nullptr;
      CUtensorMap tw = make_tmap_bf16_2d(W, N, K, bn);
      op.launch = [=](const Ptrs& T, cudaStream_t st) {
        CUtensorMap ta = make_tmap_bf16_2d(T[in], M, K, 128);
        TcEpilogue ep;
        ep.bias = b;
        ep.out = T[me];
        ep.ldo = N;
        ep.act = act;
        ep.dbg = dbg;
        ep.splits = splits;
        ep.ws = ws;
        gemm_tc_maps(ta, tw, M, N, K, bn, ep, EPI_BIAS_ACT, yb, st);
        if (splits > 1) gemm_splitk_reduce(ep, M, N, yb, st);
      };
      op.n_kernels = splits > 1 ? 2 : 1;
    } else if (!xb && !wb && !yb && tf32x3_ok(K, N) && tf32_on()) {
      // fp32 mode on the tensor cores: 3xTF32 (kernels/gemm_tf32.cu)
      const char* bn_env = getenv("DUET_GEMM_BN");
      const int bn = bn_env ? atoi(bn_env) : tf32x3_pick_bn(M, N, K, sms);
      const char* dbg_env = getenv("DUET_GEMM_DBG");  // accumulator-split experiments (gemm_tf32.cu)
      const int dbg = dbg_env ? atoi(dbg_env) : 0;
      CUtensorMap tw = make_tmap_f32_2d(W, N, K, bn);
      op.launch = [=](const Ptrs& T, cudaStream_t st) {
        CUtensorMap ta = make_tmap_f32_2d(T[in], M, K, 128);
        TcEpilogue ep;
        ep.bias = b;
        ep.out = T[me];
        ep.ldo = N;
        ep.act = act;
        ep.dbg = dbg;
        gemm_tf32x3_maps(ta, tw, M, N, K, bn, ep, EPI_BIAS_ACT, st);
      };
    } else {
      op.launch = [=](const Ptrs& T, cudaStream_t st) { gemm_simt(T[in], xb, W, wb, b, T[me], yb, M, N, K, act, st); };
    }
    if (!op.n_kernels) op.n_kernels = 1;
  } else if (n.op == "mlp") {
    if (n.arg_nodes.size() != 1 || n.params.size() < 2 || n.params.size() % 2)
      fail(DUET_EPARSE, "%" + n.name + ": mlp(%x, @W0, @b0, ...)");
    const Node& x = argn(0);
    const int L = (int)n.params.size() / 2;
    std::vector<int> dims{(int)x.shape[1]};
    std::vector<void*> Ws;
    std::vector<const float*> bs;
    int wdt = pdecl(0).dtype;
    for (int l = 0; l < L; ++l) {
      const auto& w = pdecl(2 * l);
      if (w.shape.size() != 2 || w.shape[1] != dims.back()) fail(DUET_ESHAPE, "%" + n.name + ": mlp layer shapes");
      need_dtype(n, w.dtype, wdt, "weights");
      dims.push_back((int)w.shape[0]);
      Ws.push_back(P.param(n.params[2 * l]));
      bs.push_back((const float*)P.param(n.params[2 * l + 1]));
    }
    need_dtype(n, x.dtype, wdt, "input");
    const int in = n.arg_nodes[0], M = (int)x.shape[0];
    const int act = act_code(n.attr_str("act", "relu")), last = act_code(n.attr_str("last_act", "none"));
    const int xb = x.dtype == kBF16, yb = n.dtype == kBF16;
    if (M <= 64) {
      op.launch = [=](const Ptrs& T, cudaStream_t st) {
        std::vector<const void*> w(Ws.begin(), Ws.end());
        mlp_small(T[in], xb, w.data(), bs.data(), dims.data(), L, T[me], yb, M, act, last, st);
      };
      op.n_kernels = 1;
    } else {
      std::vector<void*> mids;
      for (int l = 0; l + 1 < L; ++l) mids.push_back(P.alloc((int64_t)M * dims[l + 1] * dtype_bytes(x.dtype)));
      op.launch = [=](const Ptrs& T, cudaStream_t st) {
        const void* cur = T[in];
        for (int l = 0; l < L; ++l) {
          void* out = (l + 1 == L) ? T[me] : mids[l];
          int ob = (l + 1 == L) ? yb : xb;
          gemm_simt(cur, xb, Ws[l], xb, bs[l], out, ob, M, dims[l + 1], dims[l], l + 1 == L ? last : act, st);
          cur = out;
        }
      };
      op.n_kernels = L;
    }
  } else if (n.op == "reduce_sum") {
    nargs(1, 1);
    need_dtype(n, n.dtype, kF32, "output");
    const Node& x = argn(0);
    const int in = n.arg_nodes[0], B = (int)x.shape[0], K = (int)x.shape[1], xb = x.dtype == kBF16;
    const float* b = (const float*)P.param(n.params[0]);
    op.launch = [=](const Ptrs& T, cudaStream_t st) { reduce_sum(T[in], xb, b, (float*)T[me], B, K, st); };
    op.n_kernels = 1;
  } else if (n.op == "lstm" || n.op == "gru") {
    nargs(1, 4);
    const int kind = n.op == "lstm" ? EPI_LSTM : EPI_GRU;
    const int G = kind == EPI_LSTM ? 4 : 3;
    const Node& x = argn(0);
    const auto& wih = pdecl(0);
    const auto& whh = pdecl(1);
    if (x.shape.size() != 3) fail(DUET_ESHAPE, "%" + n.name + ": input must be [S, B, E]");
    const int S = (int)x.shape[0], B = (int)x.shape[1], E = (int)x.shape[2], H = (int)whh.shape[1];
    // seq=1: the output is every h_t, [S, B, H] time-major (a lower layer of a stacked RNN)
    const bool seq = n.attr_int("seq", 0) != 0;
    if (wih.shape[0] != G * H || wih.shape[1] != E || whh.shape[0] != G * H)
      fail(DUET_ESHAPE, "%" + n.name + ": rnn weight shapes");
    if (seq ? n.shape != std::vector<int64_t>{S, B, H} : n.shape != std::vector<int64_t>{B, H})
      fail(DUET_ESHAPE, "%" + n.name + (seq ? ": output must be [S, B, H]" : ": output must be [B, H]"));
    need_dtype(n, wih.dtype, whh.dtype, "W_ih");
    need_dtype(n, x.dtype, wih.dtype, "input");
    need_dtype(n, n.dtype, x.dtype, "output");
    const int in = n.arg_nodes[0];
    void* Wih = P.param(n.params[0]);
    void* Whh = P.param(n.params[1]);
    const float* bih = (const float*)P.param(n.params[2]);
    const float* bhh = (const float*)P.param(n.params[3]);
    const bool tc = x.dtype == kBF16 && E % 8 == 0 && H % 8 == 0;
    const int es = dtype_bytes(x.dtype);
    void* hb[2] = {P.alloc((int64_t)B * H * es), P.alloc((int64_t)B * H * es)};
    float* cst = (float*)P.alloc((int64_t)B * H * 4);
    // persistent recurrence (kernels/rnn_persist.cu): one tile per CTA when the tiles fit in half of
    // the SMs (two recurrent branches on two slots co-reside), else every SM with several tiles per
    // CTA (large batches).  DUET_RNN_PERSIST=0 forces the per-step kernels.
    static const int rp_env = getenv("DUET_RNN_PERSIST") ? atoi(getenv("DUET_RNN_PERSIST")) : 1;
    // gate-tile width: the node's tile_n attribute (a per-workload SM budget, DESIGN.md "SM sharing
    // between concurrent branches"), else DUET_RNN_BN (experiments), else automatic
    static const int rp_bn_env0 = getenv("DUET_RNN_BN") ? atoi(getenv("DUET_RNN_BN")) : 0;
    const int rp_bn_env = (int)n.attr_int("tile_n", rp_bn_env0);
    if (rp_bn_env != 0 && rp_bn_env != 64 && rp_bn_env != 128 && rp_bn_env != 256)
      fail(DUET_EINVAL, "%" + n.name + ": tile_n must be 64, 128 or 256");
    int rp_bn = 0, rp_grid = 0;
    if (tc && rp_env) {
      const int mt = (B + 127) / 128;
      for (int cand : {64, 128}) {
        if (rp_bn_env && cand != rp_bn_env) continue;
        const int tl = mt * ((H + cand / 4 - 1) / (cand / 4));
        if (tl <= sms / 2) {
          rp_bn = cand;
          rp_grid = tl;
          break;
        }
      }
      // else one tile per CTA on all SMs when 128 x 128 or 128 x 256 tiles fit (c5's LSTM256 at
      // B = 4096: 128 tiles of 128 x 256, 11.0 -> 6.8 us per step; several tiles per CTA cost about
      // one step per tile)
      for (int cand : {128, 256}) {
        const int tl = mt * ((H + cand / 4 - 1) / (cand / 4));
        if (!rp_bn && !rp_bn_env && tl <= sms) {
          rp_bn = cand;
          rp_grid = tl;
        }
      }
      if (!rp_bn) {
        // several tiles per CTA: 128 x 256 tiles (64 units; half the W bytes per FLOP of 128 x 128,
        // c5's b2/b4/b5 -9/-24/-25%) while they still outnumber the SMs (rnn_persist's bn = 256
        // path is the multi-tile one), else 128 x 128
        const int t256 = mt * ((H + 63) / 64);
        rp_bn = (rp_bn_env == 256 || !rp_bn_env) ? (t256 > sms ? 256 : 128) : rp_bn_env;
        static const int grid_env = getenv("DUET_RNN_GRID") ? atoi(getenv("DUET_RNN_GRID")) : 0;  // experiments
        // the fewest CTAs with the same most-tiles-per-CTA as all SMs: a step costs about one tile
        // per tile a CTA owns, so 256 tiles on 128 CTAs (2 each) take as long as on 148 (2 on most)
        // and leave 20 SMs to the co-running branches (c5 p50 2.77 -> 2.68 ms, measured)
        const int tl = mt * ((H + rp_bn / 4 - 1) / (rp_bn / 4));
        const int per = (tl + sms - 1) / sms;
        rp_grid = grid_env > 0 && grid_env <= sms ? grid_env : (tl + per - 1) / per;
      }
    }
    if (rp_bn) {
      const int bn = rp_bn;
      const int U = bn / 4;
      const int tiles = (H + U - 1) / U;
      const int mt = (B + 127) / 128;
      const int Np = tiles * bn;
      const int Ep = (E + 63) / 64 * 64;
      const int Kc = Ep + H;
      // several tiles per CTA with 128 x 256 tiles: the CTA-pair kernel (256 x 256 pair tiles, each
      // SM loads half the weights; DUET_RNN_PAIR=0 keeps the one-CTA kernel)
      static const int grid_env2 = getenv("DUET_RNN_GRID") ? atoi(getenv("DUET_RNN_GRID")) : 0;
      const bool pair = !grid_env2 && rnn_pair_ok(kind, bn, B, tiles, mt, sms);
      const int grid = pair ? rnn_pair_grid(tiles, mt, sms) : std::min(rp_grid, tiles * mt);
      void* Wcat = P.alloc((int64_t)Np * Kc * 2);
      float* bias = (float*)P.alloc((int64_t)Np * 4);
      // one step counter per 128-row block (the recurrence of batch rows [128 m, +128) depends on
      // those rows' h only, so a row block's step t+1 waits for its own h_t, not the whole grid)
      const int64_t ctr_bytes = ((int64_t)mt * 4 + 255) / 256 * 256;
      unsigned* counter = (unsigned*)P.alloc(ctr_bytes);
      rnn_pack(kind, Wih, Whh, bih, bhh, Wcat, bias, E, Ep, H, U, bn, tiles, 0);
      CK(cudaDeviceSynchronize());
      CUtensorMap t_w = make_tmap_bf16_2d(Wcat, Np, Kc, bn);
      // K-blocked pre-swizzled h buffers [kh][mt*128][64] (bulk-copied per k-block)
      const int64_t hs_bytes = (int64_t)((H + 63) / 64) * mt * 128 * 64 * 2;
      void* hs[2] = {P.alloc(hs_bytes), P.alloc(hs_bytes)};
      CK(cudaMemset(hs[0], 0, hs_bytes));  // units >= H of the last k-block stay zero
      CK(cudaMemset(hs[1], 0, hs_bytes));
      CUtensorMap t_h0 = make_tmap_bf16_2d(hb[0], B, H, 128), t_h1 = make_tmap_bf16_2d(hb[1], B, H, 128);
      RnnPersistArgs ra;
      ra.bias = bias;
      ra.hbuf[0] = (__nv_bfloat16*)hs[0];
      ra.hbuf[1] = (__nv_bfloat16*)hs[1];
      ra.Bp = mt * 128;
      ra.counter = counter;
      ra.c_state = cst;
      ra.S = S;
      ra.B = B;
      ra.H = H;
      ra.kx = Ep / 64;
      ra.kh = (H + 63) / 64;
      ra.tiles_n = tiles;
      ra.tiles_m = mt;
      ra.dbg = getenv("DUET_RNN_DBG") ? atoi(getenv("DUET_RNN_DBG")) : 0;
      ra.pair = pair ? 1 : 0;
      // row-block step sync (measured, tools/msync_ab.sh): several
      // tiles per CTA (c5's GRU512 14.3 -> 11.2, LSTM512 15.8 -> 11.8 us per step) and many row blocks
      // (LSTM256 at B = 4096, 32 blocks of 4 CTAs: 6.7 -> 6.3); with 2 row blocks (c3's towers) the
      // grid barrier measured faster (5.65 vs 5.87 us).  DUET_RNN_MSYNC: 0 never, 2 always.
      static const int msync_env = getenv("DUET_RNN_MSYNC") ? atoi(getenv("DUET_RNN_MSYNC")) : 1;
      const bool several = (int64_t)tiles * mt > grid;
      ra.msync = msync_env == 2 || (msync_env == 1 && (several || mt >= 4)) ? 1 : 0;
      static const int hrot_env = getenv("DUET_RNN_HROT") ? atoi(getenv("DUET_RNN_HROT")) : 1;
      ra.hrot = hrot_env;
      static const int issue2_env = getenv("DUET_RNN_ISSUE2") ? atoi(getenv("DUET_RNN_ISSUE2")) : 1;
      ra.issue2 = issue2_env;
      // one release per CTA instead of one per epilogue warp (same-address atomics at the counter's
      // L2 slice): c3 tower 393 -> 374 us, c4 GRU 587 -> 567, c5 LSTM256 424 -> 404
      // (profiles/r2_ctarel_ab.log); DUET_RNN_CTAREL=0 restores per-warp releases
      static const int ctarel_env = getenv("DUET_RNN_CTAREL") ? atoi(getenv("DUET_RNN_CTAREL")) : 1;
      ra.ctarel = ctarel_env;
      ra.wcat = Wcat;
      ra.w_rows = Np;
      ra.w_cols = Kc;
      op.launch = [=](const Ptrs& T, cudaStream_t st) {
        CK(cudaMemsetAsync(counter, 0, (size_t)mt * sizeof(unsigned), st));
        CUtensorMap tx = make_tmap_bf16_2d(T[in], (int64_t)S * B, E, 128);
        RnnPersistArgs r = ra;
        if (seq) {
          r.seq = (__nv_bfloat16*)T[me];
          r.out = r.seq + (size_t)(S - 1) * B * H;
        } else {
          r.out = (__nv_bfloat16*)T[me];
        }
        rnn_persist(kind, bn, tx, t_h0, t_h1, t_w, r, grid, st);
      };
      op.n_kernels = 1;
    } else if (tc) {
      // fused step (kernels/gemm_tc.cu EPI_LSTM/EPI_GRU): K = [x_t (E, padded to Ep) | h_{t-1} (H)],
      // 4 gate blocks per tile; no G_x buffer and no separate input-projection GEMM
      const int bn = rnn_step_bn(kind, B, H, sms);
      const int U = bn / 4;
      const int tiles = (H + U - 1) / U;
      const int Np = tiles * bn;
      const int Ep = (E + 63) / 64 * 64;
      const int Kc = Ep + H;
      void* Wcat = P.alloc((int64_t)Np * Kc * 2);
      float* bias = (float*)P.alloc((int64_t)Np * 4);
      rnn_pack(kind, Wih, Whh, bih, bhh, Wcat, bias, E, Ep, H, U, bn, tiles, 0);
      CK(cudaDeviceSynchronize());
      CUtensorMap t_w = make_tmap_bf16_2d(Wcat, Np, Kc, bn);
      CUtensorMap t_h[2] = {make_tmap_bf16_2d(hb[0], B, H, 128), make_tmap_bf16_2d(hb[1], B, H, 128)};
      op.launch = [=](const Ptrs& T, cudaStream_t st) {
        CK(cudaMemsetAsync(hb[1], 0, (size_t)B * H * es, st));
        if (kind == EPI_LSTM) CK(cudaMemsetAsync(cst, 0, (size_t)B * H * 4, st));
        CUtensorMap tx = make_tmap_bf16_2d(T[in], (int64_t)S * B, E, 128);
        for (int t = 0; t < S; ++t) {
          TcEpilogue e2;
          e2.bias = bias;
          e2.c_state = cst;
          e2.h_prev = hb[(t + 1) & 1];
          e2.h_next = (t == S - 1 && !seq) ? T[me] : hb[t & 1];
          e2.H = H;
          e2.kx = Ep / 64;
          e2.x_row0 = t * B;
          // t = 0: h_{-1} = 0, so only the x_t part of K contributes
          gemm_tc_maps(t_h[(t + 1) & 1], t_w, B, Np, t == 0 ? Ep : Kc, bn, e2, kind, 1, st, &tx);
          if (seq)
            CK(cudaMemcpyAsync((char*)T[me] + (size_t)t * B * H * es, hb[t & 1], (size_t)B * H * es,
                               cudaMemcpyDeviceToDevice, st));
        }
      };
      op.n_kernels = S;
    } else if (x.dtype == kF32 && E % 4 == 0 && H % 4 == 0 && tf32_on()) {
      // fp32 mode on the tensor cores: the fused step of the bf16 path as a 3xTF32 GEMM
      // (kernels/gemm_tf32.cu), one launch per step; x and h in fp32, K = [x_t (E, padded to 32) | h]
      const int bn = 64;
      const int U = bn / 4;
      const int tiles = (H + U - 1) / U;
      const int Np = tiles * bn;
      const int Ep = (E + 31) / 32 * 32;
      const int Kc = Ep + H;
      float* Wcat = (float*)P.alloc((int64_t)Np * Kc * 4);
      float* bias = (float*)P.alloc((int64_t)Np * 4);
      rnn_pack_f32(kind, (const float*)Wih, (const float*)Whh, bih, bhh, Wcat, bias, E, Ep, H, U, bn, tiles, 0);
      CK(cudaDeviceSynchronize());
      CUtensorMap t_w = make_tmap_f32_2d(Wcat, Np, Kc, bn);
      CUtensorMap t_h[2] = {make_tmap_f32_2d(hb[0], B, H, 128), make_tmap_f32_2d(hb[1], B, H, 128)};
      op.launch = [=](const Ptrs& T, cudaStream_t st) {
        CK(cudaMemsetAsync(hb[1], 0, (size_t)B * H * 4, st));
        if (kind == EPI_LSTM) CK(cudaMemsetAsync(cst, 0, (size_t)B * H * 4, st));
        CUtensorMap tx = make_tmap_f32_2d(T[in], (int64_t)S * B, E, 128);
        for (int t = 0; t < S; ++t) {
          TcEpilogue e2;
          e2.bias = bias;
          e2.c_state = cst;
          e2.h_prev = hb[(t + 1) & 1];
          e2.h_next = (t == S - 1 && !seq) ? T[me] : hb[t & 1];
          e2.H = H;
          e2.kx = Ep / 32;
          e2.x_row0 = t * B;
          // t = 0: h_{-1} = 0, so only the x_t part of K contributes
          gemm_tf32x3_maps(t_h[(t + 1) & 1], t_w, B, Np, t == 0 ? Ep : Kc, bn, e2, kind, st, &tx);
          if (seq)
            CK(cudaMemcpyAsync((char*)T[me] + (size_t)t * B * H * 4, hb[t & 1], (size_t)B * H * 4,
                               cudaMemcpyDeviceToDevice, st));
        }
      };
      op.n_kernels = S;
    } else {
      // fp32 parity path (original PyTorch layout): G_x = x W_ih^T + folded bias, then SIMT steps
      std::vector<int32_t> ident(G * H);
      for (int r = 0; r < G * H; ++r) ident[r] = r;
      int32_t* d_map = (int32_t*)P.alloc((int64_t)G * H * 4);
      CK(cudaMemcpy(d_map, ident.data(), (size_t)G * H * 4, cudaMemcpyHostToDevice));
      float* bias = (float*)P.alloc((int64_t)G * H * 4);
      rnn_bias_kernel<<<(G * H + 255) / 256, 256>>>(bih, bhh, d_map, bias, G * H, H, kind == EPI_GRU);
      CK(cudaGetLastError());
      const float* bhn = bhh + 2 * H;
      float* gx = (float*)P.alloc((int64_t)S * B * G * H * 4);
      const int xb = x.dtype == kBF16;
      op.launch = [=](const Ptrs& T, cudaStream_t st) {
        CK(cudaMemsetAsync(hb[1], 0, (size_t)B * H * es, st));
        if (kind == EPI_LSTM) CK(cudaMemsetAsync(cst, 0, (size_t)B * H * 4, st));
        gemm_simt(T[in], xb, Wih, xb, bias, gx, 0, S * B, G * H, E, ACT_NONE, st);
        for (int t = 0; t < S; ++t) {
          // seq: h_t goes straight into its slice of the [S, B, H] output and is read back from there
          void* hn = seq ? (char*)T[me] + (size_t)t * B * H * es : (t == S - 1) ? T[me] : hb[t & 1];
          const void* hp = (seq && t > 0) ? (const char*)T[me] + (size_t)(t - 1) * B * H * es : hb[(t + 1) & 1];
          rnn_step_simt(kind, gx + (size_t)t * B * G * H, Whh, xb, bhn, hp, hn, xb, cst, B, H, st);
        }
      };
      op.n_kernels = 1 + S;
    }
  } else if (n.op == "conv2d_bn") {
    nargs(1, 5);
    const Node& x = argn(0);
    const auto& w = pdecl(0);
    if (x.shape.size() != 4 || w.shape.size() != 4 || w.shape[3] != x.shape[3])
      fail(DUET_ESHAPE, "%" + n.name + ": conv shapes");
    need_dtype(n, x.dtype, w.dtype, "input");
    need_dtype(n, n.dtype, x.dtype, "output");
    ConvShape s{(int)x.shape[0], (int)x.shape[1], (int)x.shape[2], (int)x.shape[3], (int)w.shape[0], (int)w.shape[1],
                (int)w.shape[2], (int)n.attr_int("stride", 1), (int)n.attr_int("pad", 0), 0, 0};
    s.Ho = (s.H + 2 * s.pad - s.kh) / s.stride + 1;
    s.Wo = (s.W + 2 * s.pad - s.kw) / s.stride + 1;
    if (n.shape != std::vector<int64_t>{s.N, s.Ho, s.Wo, s.Co}) fail(DUET_ESHAPE, "%" + n.name + ": conv output shape");
    const int bf = x.dtype == kBF16;
    int act = act_code(n.attr_str("act", "none"));
    const int64_t per_co = (int64_t)s.kh * s.kw * s.C;
    const int in = n.arg_nodes[0];
    // residual fusion (planned in ensure_program): write act(conv + bias + res) into the add's buffer
    int res = -1, dst = me;
    auto fz = P.fuse_res.find(me);
    if (fz != P.fuse_res.end()) {
      res = fz->second.first;
      dst = fz->second.second;
      act = act_code(g.nodes[dst].attr_str("act", "none"));
    }
    // bf16 paths: C % 64 == 0 -> persistent TMA-im2col implicit GEMM; otherwise (the 3-channel
    // stem) explicit im2col [M, ldk] + the CTA-pair GEMM with the folded BN as its bias.
    static const bool no_stem = getenv("DUET_CONV_STEM") && atoi(getenv("DUET_CONV_STEM")) == 0;
    const bool tma = bf && s.Co % 16 == 0 && conv_tma_ok(s);
    const bool stem = bf && !tma && res < 0 && !no_stem && conv_stem_ok(s);
    const bool cols = bf && !tma && !stem && s.Co >= 16 && s.Co % 8 == 0 && res < 0;
    // fp32 mode on the tensor cores (3xTF32, gemm_tf32.cu): implicit GEMM with im2col TMA when
    // C % 32 == 0, else (the stem) explicit im2col + the 3xTF32 GEMM
    const bool f32tc = !bf && tf32_on() && conv_tf32_ok(s);
    const bool f32cols = !bf && tf32_on() && !f32tc && s.Co >= 16 && s.Co % 4 == 0 && res < 0;
    const int64_t ldw = (tma || cols || stem) ? (per_co + 7) / 8 * 8 : f32cols ? (per_co + 3) / 4 * 4 : per_co;
    void* Wf = P.alloc((int64_t)s.Co * ldw * dtype_bytes(w.dtype));
    float* bias = (float*)P.alloc((int64_t)s.Co * 4);
    fold_bn(P.param(n.params[0]), bf, (const float*)P.param(n.params[1]), (const float*)P.param(n.params[2]),
            (const float*)P.param(n.params[3]), (const float*)P.param(n.params[4]), Wf, bias, s.Co, per_co, ldw, 0);
    static const bool conv_dyn = !(getenv("DUET_CONV_DYN") && atoi(getenv("DUET_CONV_DYN")) == 0);
    if (tma) {
      ConvPlan plan = conv_tc_plan(s, sms);
      if (const char* f = getenv("DUET_CONV_BN")) {  // tile-width sweeps (tools/plan_sweep.sh)
        const int fb = atoi(f);
        if (fb == 64 || fb == 128 || fb == 256) plan.bn = fb;
      }
      CUtensorMap tw = make_tmap_bf16_2d(Wf, s.Co, ldw, plan.bn);
      const int K = (int)per_co;
      // dynamic tile scheduling (DUET_CONV_DYN=0: static persistent tiles)
      unsigned* ctr = nullptr;
      if (conv_dyn) {
        ctr = (unsigned*)P.alloc(2 * sizeof(unsigned));
        CK(cudaMemset(ctr, 0, 2 * sizeof(unsigned)));
      }
      op.launch = [=](const Ptrs& T, cudaStream_t st) {
        conv_tc(tw, T[in], bias, res >= 0 ? T[res] : nullptr, T[dst], s, K, act, plan, ctr, st);
      };
      op.n_kernels = 1;
    } else if (f32tc) {
      const int bn = tf32x3_pick_bn((int)std::min<int64_t>((int64_t)s.N * s.Ho * s.Wo, INT32_MAX), s.Co,
                                    conv_taps(s).nr * conv_taps(s).ns * s.C, sms);
      CUtensorMap tw = make_tmap_f32_2d(Wf, s.Co, ldw, bn);
      op.launch = [=](const Ptrs& T, cudaStream_t st) {
        conv_tf32x3(tw, T[in], bias, res >= 0 ? T[res] : nullptr, T[dst], s, act, bn, st);
      };
      op.n_kernels = 1;
    } else if (f32cols) {
      const int64_t M = (int64_t)s.N * s.Ho * s.Wo;
      void* colbuf = P.alloc(M * ldw * 4);
      const int bn = tf32x3_pick_bn((int)M, s.Co, (int)ldw, sms);
      CUtensorMap tw = make_tmap_f32_2d(Wf, s.Co, ldw, bn);
      CUtensorMap ta = make_tmap_f32_2d(colbuf, M, ldw, 128);
      op.launch = [=](const Ptrs& T, cudaStream_t st) {
        im2col_f32(T[in], colbuf, s, ldw, st);
        TcEpilogue ep;
        ep.bias = bias;
        ep.out = T[dst];
        ep.ldo = s.Co;
        ep.act = act;
        gemm_tf32x3_maps(ta, tw, (int)M, s.Co, (int)ldw, bn, ep, EPI_BIAS_ACT, st);
      };
      op.n_kernels = 2;
    } else if (stem) {
      void* Wk = P.alloc((int64_t)s.Co * 192 * 2);
      conv_stem_pack(Wf, ldw, Wk, s, 0);
      CUtensorMap tw = conv_stem_wmap(Wk, s.Co);
      unsigned* ctr = nullptr;
      if (conv_dyn) {
        ctr = (unsigned*)P.alloc(2 * sizeof(unsigned));
        CK(cudaMemset(ctr, 0, 2 * sizeof(unsigned)));
      }
      op.launch = [=](const Ptrs& T, cudaStream_t st) { conv_stem(tw, T[in], bias, T[dst], s, act, ctr, st); };
      op.n_kernels = 1;
    } else if (cols) {
      const int64_t M = (int64_t)s.N * s.Ho * s.Wo;
      void* colbuf = P.alloc(M * ldw * 2);
      const int bn = tc2_pick_bn((int)M, s.Co, (int)ldw, sms);
      CUtensorMap tw = make_tmap_bf16_2d(Wf, s.Co, ldw, bn / 2);
      CUtensorMap ta = make_tmap_bf16_2d(colbuf, M, ldw, 128);
      op.launch = [=](const Ptrs& T, cudaStream_t st) {
        im2col(T[in], colbuf, s, ldw, st);
        TcEpilogue ep;
        ep.bias = bias;
        ep.out = T[dst];
        ep.ldo = s.Co;
        ep.act = act;
        gemm_tc2_maps(ta, tw, (int)M, s.Co, (int)ldw, bn, ep, 1, st);
      };
      op.n_kernels = 2;
    } else {
      op.launch = [=](const Ptrs& T, cudaStream_t st) {
        conv_fwd(T[in], Wf, bias, res >= 0 ? T[res] : nullptr, T[dst], bf, s, act, st);
      };
      op.n_kernels = 1;
    }
  } else if (n.op == "add") {
    nargs(2, 0);
    if (P.fused_adds.count(me)) return;  // computed by the fused conv epilogue
    need_dtype(n, argn(0).dtype, n.dtype, "a");
    need_dtype(n, argn(1).dtype, n.dtype, "b");
    if (argn(0).numel() != n.numel() || argn(1).numel() != n.numel()) fail(DUET_ESHAPE, "%" + n.name + ": add shapes");
    const int a = n.arg_nodes[0], b = n.arg_nodes[1], bf = n.dtype == kBF16;
    const int act = act_code(n.attr_str("act", "none"));
    const int64_t cnt = n.numel();
    op.launch = [=](const Ptrs& T, cudaStream_t st) { add_act(T[a], T[b], T[me], bf, cnt, act, st); };
    op.n_kernels = 1;
  } else if (n.op == "sigmoid") {
    nargs(1, 0);
    need_dtype(n, argn(0).dtype, n.dtype, "input");
    const int a = n.arg_nodes[0], bf = n.dtype == kBF16;
    const int64_t cnt = n.numel();
    op.launch = [=](const Ptrs& T, cudaStream_t st) { sigmoid_ew(T[a], T[me], bf, cnt, st); };
    op.n_kernels = 1;
  } else if (n.op == "bert_embed") {
    // MT-DNN lexicon encoder: [B*S, H] = LN(E_tok[tok] + E_pos[s] + E_seg[seg])
    nargs(2, 5);
    need_dtype(n, argn(0).dtype, kI32, "tokens");
    need_dtype(n, argn(1).dtype, kI32, "segments");
    const auto& et = pdecl(0);
    const auto& ep_ = pdecl(1);
    const auto& es = pdecl(2);
    need_dtype(n, n.dtype, et.dtype, "output");
    need_dtype(n, ep_.dtype, et.dtype, "position table");
    need_dtype(n, es.dtype, et.dtype, "segment table");
    if (argn(0).shape.size() != 2 || argn(1).shape != argn(0).shape) fail(DUET_ESHAPE, "%" + n.name + ": tokens [B, S]");
    const int B = (int)argn(0).shape[0], S = (int)argn(0).shape[1], H = (int)et.shape[1];
    if (et.shape.size() != 2 || ep_.shape.size() != 2 || es.shape.size() != 2 || ep_.shape[0] < S ||
        ep_.shape[1] != H || es.shape[1] != H || pdecl(3).numel() != H || pdecl(4).numel() != H ||
        n.shape != std::vector<int64_t>{(int64_t)B * S, H})
      fail(DUET_ESHAPE, "%" + n.name + ": bert_embed shapes");
    const int a0 = n.arg_nodes[0], a1 = n.arg_nodes[1], bf = n.dtype == kBF16;
    const void *Et = P.param(n.params[0]), *Ep = P.param(n.params[1]), *Es = P.param(n.params[2]);
    const float* gm = (const float*)P.param(n.params[3]);
    const float* bt = (const float*)P.param(n.params[4]);
    const int64_t V = et.shape[0];
    op.launch = [=](const Ptrs& T, cudaStream_t st) {
      bert_embed((const int32_t*)T[a0], (const int32_t*)T[a1], Et, Ep, Es, gm, bt, T[me], bf, B, S, H, V, st);
    };
    op.n_kernels = 1;
  } else if (n.op == "attention") {
    nargs(1, 0);
    const Node& x = argn(0);
    need_dtype(n, x.dtype, n.dtype, "qkv");
    const int heads = (int)n.attr_int("heads", 0), S = (int)n.attr_int("seq", 0);
    if (x.shape.size() != 2 || heads <= 0 || S <= 0 || x.shape[0] % S || x.shape[1] % (3 * heads) ||
        n.shape != std::vector<int64_t>{x.shape[0], x.shape[1] / 3})
      fail(DUET_ESHAPE, "%" + n.name + ": attention needs qkv [B*S, 3H] and output [B*S, H]");
    const int B = (int)(x.shape[0] / S), dh = (int)(x.shape[1] / 3 / heads);
    if (!attention_ok(S, dh)) fail(DUET_EUNSUPPORTED, "%" + n.name + ": attention needs S <= 512, dh in {32, 64, 128}, K and V in shared memory");
    const int a = n.arg_nodes[0], bf = n.dtype == kBF16;
    static const bool no_att_tc = getenv("DUET_ATT_TC") && atoi(getenv("DUET_ATT_TC")) == 0;
    if (attention_tc_ok(S, dh, bf) && !no_att_tc)
      op.launch = [=](const Ptrs& T, cudaStream_t st) { attention_tc(T[a], T[me], B, S, heads, st); };
    else
      op.launch = [=](const Ptrs& T, cudaStream_t st) { attention(T[a], T[me], bf, B, S, heads, dh, st); };
    op.n_kernels = 1;
  } else if (n.op == "add_layernorm") {
    nargs(2, 2);
    need_dtype(n, argn(0).dtype, n.dtype, "a");
    need_dtype(n, argn(1).dtype, n.dtype, "b");
    if (argn(0).shape != n.shape || argn(1).shape != n.shape || n.shape.size() != 2 ||
        pdecl(0).numel() != n.shape[1] || pdecl(1).numel() != n.shape[1])
      fail(DUET_ESHAPE, "%" + n.name + ": add_layernorm shapes");
    const int a = n.arg_nodes[0], b = n.arg_nodes[1], bf = n.dtype == kBF16, H = (int)n.shape[1];
    const int64_t rows = n.shape[0];
    const float* gm = (const float*)P.param(n.params[0]);
    const float* bt = (const float*)P.param(n.params[1]);
    op.launch = [=](const Ptrs& T, cudaStream_t st) { add_layernorm(T[a], T[b], gm, bt, T[me], bf, rows, H, st); };
    op.n_kernels = 1;
  } else if (n.op == "select_rows") {
    nargs(1, 0);
    const Node& x = argn(0);
    need_dtype(n, x.dtype, n.dtype, "input");
    const int64_t stride = n.attr_int("stride", 1), offset = n.attr_int("offset", 0);
    if (x.shape.size() != 2 || n.shape.size() != 2 || n.shape[1] != x.shape[1] || stride < 1 || offset < 0 ||
        offset + (n.shape[0] - 1) * stride >= x.shape[0])
      fail(DUET_ESHAPE, "%" + n.name + ": select_rows shapes");
    const int a = n.arg_nodes[0], es = dtype_bytes(n.dtype);
    const int64_t rows = n.shape[0], cols = n.shape[1];
    op.launch = [=](const Ptrs& T, cudaStream_t st) { select_rows(T[a], T[me], es, rows, cols, stride, offset, st); };
    op.n_kernels = 1;
  } else if (n.op == "maxpool") {
    nargs(1, 0);
    const Node& x = argn(0);
    need_dtype(n, x.dtype, n.dtype, "input");
    const int a = n.arg_nodes[0], bf = n.dtype == kBF16;
    const int N = (int)x.shape[0], H = (int)x.shape[1], W = (int)x.shape[2], C = (int)x.shape[3];
    const int k = (int)n.attr_int("k", 3), s = (int)n.attr_int("stride", 2), p = (int)n.attr_int("pad", 1);
    const int Ho = (H + 2 * p - k) / s + 1, Wo = (W + 2 * p - k) / s + 1;
    if (n.shape != std::vector<int64_t>{N, Ho, Wo, C}) fail(DUET_ESHAPE, "%" + n.name + ": maxpool output shape");
    op.launch = [=](const Ptrs& T, cudaStream_t st) { maxpool_nhwc(T[a], T[me], bf, N, H, W, C, k, s, p, Ho, Wo, st); };
    op.n_kernels = 1;
  } else if (n.op == "avgpool") {
    nargs(1, 0);
    const Node& x = argn(0);
    need_dtype(n, x.dtype, n.dtype, "input");
    const int a = n.arg_nodes[0], bf = n.dtype == kBF16;
    const int N = (int)x.shape[0], H = (int)x.shape[1], W = (int)x.shape[2], C = (int)x.shape[3];
    op.launch = [=](const Ptrs& T, cudaStream_t st) { avgpool_nhwc(T[a], T[me], bf, N, H, W, C, st); };
    op.n_kernels = 1;
  } else if (n.op == "dot_join") {
    nargs(2, 2);
    need_dtype(n, argn(0).dtype, kF32, "wide logit");
    need_dtype(n, n.dtype, kF32, "output");
    const Node& a = argn(1);
    const int s = n.arg_nodes[0], ai = n.arg_nodes[1], B = (int)a.shape[0], K = (int)a.shape[1];
    const int ab = a.dtype == kBF16;
    const float* w = (const float*)P.param(n.params[0]);
    const float* b = (const float*)P.param(n.params[1]);
    op.launch = [=](const Ptrs& T, cudaStream_t st) {
      dot_join((const float*)T[s], T[ai], ab, w, b, (float*)T[me], B, K, st);
    };
    op.n_kernels = 1;
  } else if (n.op == "cosine_join") {
    nargs(2, 0);
    need_dtype(n, argn(1).dtype, argn(0).dtype, "b");
    need_dtype(n, n.dtype, kF32, "output");
    const int a = n.arg_nodes[0], b = n.arg_nodes[1], B = (int)argn(0).shape[0], K = (int)argn(0).shape[1];
    const int bf = argn(0).dtype == kBF16;
    op.launch = [=](const Ptrs& T, cudaStream_t st) { cosine_join(T[a], T[b], bf, (float*)T[me], B, K, st); };
    op.n_kernels = 1;
  } else if (n.op == "concat_head") {
    if (n.params.size() != 2 || n.arg_nodes.empty()) fail(DUET_EPARSE, "%" + n.name + ": concat_head(%a..., @w, @b)");
    need_dtype(n, n.dtype, kF32, "output");
    std::vector<int> ins, Ks, bfs;
    int64_t tot = 0;
    for (size_t i = 0; i < n.arg_nodes.size(); ++i) {
      ins.push_back(n.arg_nodes[i]);
      Ks.push_back((int)argn(i).shape[1]);
      bfs.push_back(argn(i).dtype == kBF16);
      tot += Ks.back();
    }
    if (pdecl(0).numel() != tot) fail(DUET_ESHAPE, "%" + n.name + ": head weight length != concat width");
    const int B = (int)n.shape[0], act = act_code(n.attr_str("act", "sigmoid"));
    const float* w = (const float*)P.param(n.params[0]);
    const float* b = (const float*)P.param(n.params[1]);
    op.launch = [=](const Ptrs& T, cudaStream_t st) {
      std::vector<const void*> parts;
      for (int i : ins) parts.push_back(T[i]);
      concat_head(parts.data(), Ks.data(), bfs.data(), (int)ins.size(), w, b, (float*)T[me], B, act, st);
    };
    op.n_kernels = 1;
  } else if (n.op == "sum_join" || n.op == "mean_join") {
    if (!n.params.empty() || n.arg_nodes.empty()) fail(DUET_EPARSE, "%" + n.name + ": logit join arguments");
    need_dtype(n, n.dtype, kF32, "output");
    std::vector<int> ins(n.arg_nodes.begin(), n.arg_nodes.end());
    for (size_t i = 0; i < ins.size(); ++i) need_dtype(n, argn(i).dtype, kF32, "branch logit");
    const int B = (int)n.shape[0], mean = n.op == "mean_join";
    op.launch = [=](const Ptrs& T, cudaStream_t st) {
      std::vector<const float*> parts;
      for (int i : ins) parts.push_back((const float*)T[i]);
      logit_join(parts.data(), (int)parts.size(), (float*)T[me], B, mean, st);
    };
    op.n_kernels = 1;
  } else {
    fail(DUET_EUNSUPPORTED, "%" + n.name + ": no kernel for operator '" + n.op + "'");
  }
}

// add(%a, %b){act} whose later operand (topological rank) is a conv2d_bn with act=none consumed
// only by this add: the conv's epilogue adds the other operand and applies the add's activation,
// writing the add's buffer (ResNet BasicBlock tail; no extra HBM round trip).
void plan_residual_fusion(Program& P) {
  const Graph& g = *P.g;
  std::vector<int> rank(g.nodes.size());
  for (size_t i = 0; i < g.topo.size(); ++i) rank[g.topo[i]] = (int)i;
  std::vector<int> n_cons(g.nodes.size(), 0);
  for (auto& n : g.nodes)
    for (int u : n.inputs) n_cons[u]++;
  std::set<int> outs(g.outputs.begin(), g.outputs.end());
  for (auto& n : g.nodes) {
    if (n.op != "add" || n.arg_nodes.size() != 2 || n.arg_nodes[0] == n.arg_nodes[1]) continue;
    int a = n.arg_nodes[0], b = n.arg_nodes[1];
    int late = rank[a] > rank[b] ? a : b, other = late == a ? b : a;
    const Node& c = g.nodes[late];
    if (c.op != "conv2d_bn" || c.attr_str("act", "none") != "none" || n_cons[late] != 1 || outs.count(late)) continue;
    if (c.dtype != kBF16 || n.dtype != kBF16 || c.shape != n.shape || g.nodes[other].shape != n.shape) continue;
    if (c.shape.size() != 4 || c.shape[3] % 16) continue;
    P.fuse_res[late] = {other, n.id};
    P.fused_adds.insert(n.id);
  }
}


std::shared_ptr<Program> ensure_program(Graph* g) {
  if (g->prog) return g->prog;
  for (auto& name : g->param_order)
    if (!g->bound.count(name)) fail(DUET_EUNBOUND, "parameter @" + name + " is not bound");
  int dev = 0;
  if (!g->bound.empty())
    dev = g->bound.begin()->second.device;
  else
    CK(cudaGetDevice(&dev));
  DeviceGuard dg(dev);
  auto P = std::make_shared<Program>();
  P->g = g;
  P->device = dev;
  P->buf.resize(g->nodes.size(), nullptr);
  for (auto& n : g->nodes) P->buf[n.id] = P->alloc(n.nbytes());
  P->ops.resize(g->nodes.size());
  plan_residual_fusion(*P);
  for (auto& n : g->nodes) build_op(*P, n, P->ops[n.id]);
  CK(cudaDeviceSynchronize());
  g->prog = P;
  return P;
}

void launch_subgraph(const Program& P, const Partition& part, int s, const Ptrs& T, cudaStream_t st) {
  for (int v : part.sg_nodes[s])
    if (P.ops[v].launch) P.ops[v].launch(T, st);
}

int subgraph_kernels(const Program& P, const Partition& part, int s) {
  int nk = 0;
  for (int v : part.sg_nodes[s]) nk += P.ops[v].n_kernels;
  return nk;
}

int64_t tensor_numel(const duet_tensor& t) {
  int64_t n = 1;
  for (int i = 0; i < t.ndim; ++i) n *= t.shape[i];
  return n;
}

void check_tensor(const Node& n, const duet_tensor& t, const char* what) {
  if ((int)t.dtype != n.dtype)
    fail(DUET_EDTYPE, std::string(what) + " %" + n.name + ": dtype " + dtype_name(t.dtype) + " != " + dtype_name(n.dtype));
  if (t.ndim != (int)n.shape.size()) fail(DUET_ESHAPE, std::string(what) + " %" + n.name + ": rank mismatch");
  for (int i = 0; i < t.ndim; ++i)
    if (t.shape[i] != n.shape[i]) fail(DUET_ESHAPE, std::string(what) + " %" + n.name + ": shape mismatch");
  if (!t.data && n.numel() > 0) fail(DUET_EINVAL, std::string(what) + " %" + n.name + ": NULL data");
}

}  // namespace

// ------------------------------------------------------------------------------------------------
// Executor
// ------------------------------------------------------------------------------------------------
struct ExecEntry {
  std::vector<void*> key;
  cudaGraph_t graph = nullptr;
  cudaGraphExec_t exec = nullptr;
  std::vector<cudaEvent_t> events;
  // trace (Schedule::trace): timing events at the fork and around every subgraph (also in events),
  // recorded as external event-record nodes of the graph (a plain record during capture only
  // expresses a dependency)
  cudaEvent_t t_fork = nullptr;
  std::vector<cudaEvent_t> t_start, t_end;
};

struct ExecCache {
  int device = 0;
  std::vector<ExecEntry> entries;
  int64_t launches = 0;
  int last = -1;  // entry of the last duet_run (trace export)
  std::weak_ptr<Program> prog;
  ~ExecCache() {
    int prev = 0;
    cudaGetDevice(&prev);
    cudaSetDevice(device);
    for (auto& e : entries) {
      if (e.exec) cudaGraphExecDestroy(e.exec);
      if (e.graph) cudaGraphDestroy(e.graph);
      for (auto ev : e.events) cudaEventDestroy(ev);
    }
    cudaSetDevice(prev);
  }
};

void destroy_exec(ExecCache* e) { delete e; }

struct HostCopy {
  void* dst;
  const void* src;
  size_t bytes;
  cudaMemcpyKind kind;
  int node = -1;  // H2D: the input node it fills (its consumers wait on the copy's event)
};

static ExecEntry capture(const Program& P, const Schedule& S, const std::vector<cudaStream_t>& streams,
                         const Ptrs& T, const std::vector<HostCopy>& h2d, const std::vector<HostCopy>& d2h,
                         int64_t* launches) {
  const Partition& part = *S.p;
  ExecEntry E;
  cudaStream_t home = streams[0];
  const int n = part.n_sg();
  auto mk = [&]() {
    cudaEvent_t ev;
    CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
    E.events.push_back(ev);
    return ev;
  };
  std::vector<cudaEvent_t> done(n);
  for (int s = 0; s < n; ++s) done[s] = mk();
  cudaEvent_t fork = mk();
  auto mk_timed = [&]() {
    cudaEvent_t ev;
    CK(cudaEventCreate(&ev));
    E.events.push_back(ev);
    return ev;
  };
  if (S.trace) {
    E.t_fork = mk_timed();
    for (int s = 0; s < n; ++s) {
      E.t_start.push_back(mk_timed());
      E.t_end.push_back(mk_timed());
    }
  }
  // subgraph-level predecessors
  std::vector<std::vector<int>> preds(n);
  for (auto& kv : part.edges)
    if (kv.first.first >= 0 && kv.first.second >= 0) preds[kv.first.second].push_back(kv.first.first);
  // H2D copies of pinned-host inputs start at the fork, each on its own side stream (one memcpy
  // node + one event per input), so every copy overlaps all branch compute from t = 0 and a small
  // input never queues behind a large one (c4's token ids vs its 19 MB image); each consuming
  // subgraph waits only on the events of the inputs it reads.
  const Graph& G = *part.g;
  std::vector<std::vector<int>> copies_of(n);  // subgraph -> indices into h2d it consumes
  for (size_t c = 0; c < h2d.size(); ++c) {
    if (h2d[c].node < 0) continue;
    for (int s = 0; s < n; ++s)
      for (int v : part.sg_nodes[s]) {
        const auto& an = G.nodes[v].arg_nodes;
        if (std::find(an.begin(), an.end(), h2d[c].node) != an.end()) {
          copies_of[s].push_back((int)c);
          break;
        }
      }
  }
  std::vector<cudaEvent_t> copied(h2d.size(), nullptr);
  std::vector<cudaStream_t> side(h2d.size(), nullptr);
  for (auto& st : side) CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  auto free_side = [&]() {
    for (auto st : side)
      if (st) cudaStreamDestroy(st);
  };
  int64_t nk = 0;
  CK(cudaStreamBeginCapture(home, cudaStreamCaptureModeRelaxed));
  try {
    CK(cudaEventRecord(fork, home));
    if (S.trace) CK(cudaEventRecordWithFlags(E.t_fork, home, cudaEventRecordExternal));
    // pinned-host inputs/outputs are memcpy nodes of the same graph: one launch per inference
    for (size_t c = 0; c < h2d.size(); ++c) {
      CK(cudaStreamWaitEvent(side[c], fork, 0));
      CK(cudaMemcpyAsync(h2d[c].dst, h2d[c].src, h2d[c].bytes, h2d[c].kind, side[c]));
      copied[c] = mk();
      CK(cudaEventRecord(copied[c], side[c]));
    }
    std::vector<char> forked(streams.size(), 0);
    std::vector<int> last_on(streams.size(), -1);
    for (int s : S.order) {
      const int d = S.slot_of[s];
      cudaStream_t st = streams[d];
      // slot index of the first slot that uses this stream handle (aliases share a queue)
      int q = d;
      for (int k = 0; k < (int)streams.size(); ++k)
        if (streams[k] == st) {
          q = k;
          break;
        }
      if (st != home && !forked[q]) {
        CK(cudaStreamWaitEvent(st, fork, 0));
        forked[q] = 1;
      }
      for (int u : preds[s])
        if (streams[S.slot_of[u]] != st) CK(cudaStreamWaitEvent(st, done[u], 0));
      for (int c : copies_of[s]) CK(cudaStreamWaitEvent(st, copied[c], 0));
      if (S.trace) CK(cudaEventRecordWithFlags(E.t_start[s], st, cudaEventRecordExternal));
      launch_subgraph(P, part, s, T, st);
      nk += subgraph_kernels(P, part, s);
      if (S.trace) CK(cudaEventRecordWithFlags(E.t_end[s], st, cudaEventRecordExternal));
      CK(cudaEventRecord(done[s], st));
      last_on[q] = s;
    }
    for (size_t q = 0; q < streams.size(); ++q)
      if (last_on[q] >= 0 && streams[q] != home) CK(cudaStreamWaitEvent(home, done[last_on[q]], 0));
    for (auto ev : copied) CK(cudaStreamWaitEvent(home, ev, 0));  // joins every side stream
    for (auto& c : d2h) CK(cudaMemcpyAsync(c.dst, c.src, c.bytes, c.kind, home));
  } catch (...) {
    cudaGraph_t junk = nullptr;
    cudaStreamEndCapture(home, &junk);
    if (junk) cudaGraphDestroy(junk);
    cudaGetLastError();
    for (auto ev : E.events) cudaEventDestroy(ev);
    free_side();
    throw;
  }
  CK(cudaStreamEndCapture(home, &E.graph));
  free_side();
  static const bool log = getenv("DUET_MEASURE_LOG") != nullptr;
  auto t_inst = std::chrono::steady_clock::now();
  // per-node priorities: kernels captured from a higher-priority slot stream keep it inside the
  // graph, so a latency-bound branch gets SMs first when a co-running branch's CTAs retire
  CK(cudaGraphInstantiate(&E.exec, E.graph, cudaGraphInstantiateFlagUseNodePriority));
  if (log) {
    size_t nn = 0;
    cudaGraphGetNodes(E.graph, nullptr, &nn);
    fprintf(stderr, "[capture] %zu graph nodes, instantiate %.1f ms\n", nn,
            std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_inst).count());
  }
  *launches = nk;
  return E;
}

// ---- zero-copy host I/O (duet_run with pinned HOST tensors) ----------------------------------
// A pinned host buffer is device-addressable (UVA).  An input whose single consumer reads it once,
// coalesced (hashing, the id reads of the gathers), is read by that kernel over PCIe: no copy
// engine round trip, and the transfer overlaps the kernel's own work.  An output nobody in the
// graph reads, produced by a plain-store kernel (the joins), is stored straight into host memory.
// Everything else (pageable memory, several consumers, strided / re-read access such as token
// ids or conv images) keeps the memcpy nodes.  DUET_ZERO_COPY=0 disables both.
static bool zero_copy_enabled() {
  static const bool on = !(getenv("DUET_ZERO_COPY") && atoi(getenv("DUET_ZERO_COPY")) == 0);
  return on;
}

static void* mapped_host_ptr(const void* p) {
  cudaPointerAttributes a{};
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  if (a.type != cudaMemoryTypeHost || !a.devicePointer) return nullptr;
  return a.devicePointer;
}

static void* direct_input_ptr(const Graph& g, const Node& in, const void* host) {
  if (!zero_copy_enabled()) return nullptr;
  const Node* consumer = nullptr;
  int uses = 0;
  for (const Node& c : g.nodes)
    for (int a : c.arg_nodes)
      if (a == in.id) ++uses, consumer = &c;
  for (int o : g.outputs)
    if (o == in.id) return nullptr;
  if (uses != 1) return nullptr;
  const std::string& op = consumer->op;
  if (op != "hash_mod" && op != "gather_sum" && op != "gather_concat") return nullptr;
  return mapped_host_ptr(host);
}

static void* direct_output_ptr(const Graph& g, const Node& out, void* host) {
  if (!zero_copy_enabled()) return nullptr;
  for (const Node& c : g.nodes)
    for (int a : c.arg_nodes)
      if (a == out.id) return nullptr;
  int listed = 0;
  for (int o : g.outputs) listed += o == out.id;
  if (listed != 1) return nullptr;
  static const char* ok[] = {"dot_join", "cosine_join", "concat_head", "sum_join", "mean_join", "reduce_sum", "gather_sum"};
  bool found = false;
  for (auto* k : ok) found |= out.op == k;
  if (!found) return nullptr;
  return mapped_host_ptr(host);
}

void run_schedule(Schedule* S, const duet_slot* slots, int n_slots, const duet_tensor* in, int n_in, duet_tensor* out,
                  int n_out) {
  const Graph* gc = S->p->g;
  Graph* g = const_cast<Graph*>(gc);
  auto P = ensure_program(g);
  if (n_slots != S->pr->n_slots) fail(DUET_EINVAL, "n_slots differs from the profile's slot count");
  std::vector<cudaStream_t> streams;
  for (int d = 0; d < n_slots; ++d) {
    if (slots[d].gpu != P->device)
      fail(DUET_EUNSUPPORTED, "slot on another GPU: this build runs one GPU per process (multi-GPU = ranks)");
    if (!slots[d].stream) fail(DUET_EINVAL, "slot stream is NULL (the legacy default stream cannot be captured)");
    streams.push_back((cudaStream_t)slots[d].stream);
  }
  if (n_in != (int)g->input_nodes.size()) fail(DUET_EINVAL, "wrong number of inputs");
  if (n_out != (int)g->outputs.size()) fail(DUET_EINVAL, "wrong number of outputs");
  DeviceGuard dg(P->device);
  cudaStream_t home = streams[0];
  Ptrs T = P->buf;
  std::vector<HostCopy> h2d, d2h;
  for (int i = 0; i < n_in; ++i) {
    const Node& nd = g->nodes[g->input_nodes[i]];
    check_tensor(nd, in[i], "input");
    if (in[i].device >= 0) {
      if (in[i].device != P->device) fail(DUET_EUNSUPPORTED, "input on another GPU");
      T[nd.id] = in[i].data;
    } else if (!mapped_host_ptr(in[i].data)) {
      fail(DUET_EINVAL, "input " + nd.name + ": host tensors must be pinned (page-locked) memory");
    } else if (void* dp = direct_input_ptr(*g, nd, in[i].data)) {
      T[nd.id] = dp;  // zero-copy: its only consumer streams it once over PCIe
    } else {
      h2d.push_back({P->buf[nd.id], in[i].data, (size_t)nd.nbytes(), cudaMemcpyHostToDevice, nd.id});
    }
  }
  for (int i = 0; i < n_out; ++i) {
    const Node& nd = g->nodes[g->outputs[i]];
    check_tensor(nd, out[i], "output");
    if (out[i].device >= 0) {
      if (out[i].device != P->device) fail(DUET_EUNSUPPORTED, "output on another GPU");
      T[nd.id] = out[i].data;
    } else if (!mapped_host_ptr(out[i].data)) {
      fail(DUET_EINVAL, "output " + nd.name + ": host tensors must be pinned (page-locked) memory");
    } else if (void* dp = direct_output_ptr(*g, nd, out[i].data)) {
      T[nd.id] = dp;  // zero-copy: the producing kernel stores straight into pinned host memory
    } else {
      d2h.push_back({out[i].data, P->buf[nd.id], (size_t)nd.nbytes(), cudaMemcpyDeviceToHost});
    }
  }
  if (!S->exec || S->exec->prog.lock() != P) {
    S->exec = std::make_shared<ExecCache>();
    S->exec->device = P->device;
    S->exec->prog = P;
  }
  std::vector<void*> key(T.begin(), T.end());
  for (auto st : streams) key.push_back((void*)st);
  for (auto& c : h2d) key.push_back(const_cast<void*>(c.src));
  for (auto& c : d2h) key.push_back(c.dst);
  key.push_back((void*)(intptr_t)S->trace);
  ExecEntry* hit = nullptr;
  for (auto& e : S->exec->entries)
    if (e.key == key) hit = &e;
  if (!hit) {
    int64_t nk = 0;
    ExecEntry E = capture(*P, *S, streams, T, h2d, d2h, &nk);
    E.key = key;
    S->exec->launches = nk;
    if (S->exec->entries.size() >= 8) {
      auto& old = S->exec->entries.front();
      cudaGraphExecDestroy(old.exec);
      cudaGraphDestroy(old.graph);
      for (auto ev : old.events) cudaEventDestroy(ev);
      S->exec->entries.erase(S->exec->entries.begin());
    }
    S->exec->entries.push_back(std::move(E));
    hit = &S->exec->entries.back();
  }
  S->exec->last = (int)(hit - S->exec->entries.data());
  CK(cudaGraphLaunch(hit->exec, home));
}

void schedule_trace_export(const Schedule* s, int64_t* start_ns, int64_t* end_ns, int n) {
  if (!s->exec || s->exec->last < 0) fail(DUET_ESTATE, "no duet_run of this schedule yet");
  const ExecEntry& E = s->exec->entries[s->exec->last];
  if (!E.t_fork) fail(DUET_ESTATE, "the last duet_run was not traced (duet_schedule_set_trace)");
  if (n != (int)E.t_start.size()) fail(DUET_EINVAL, "trace: n must equal the subgraph count");
  DeviceGuard dg(s->exec->device);
  for (int i = 0; i < n; ++i) {
    CK(cudaEventSynchronize(E.t_end[i]));
    float a = 0, b = 0;
    CK(cudaEventElapsedTime(&a, E.t_fork, E.t_start[i]));
    CK(cudaEventElapsedTime(&b, E.t_fork, E.t_end[i]));
    if (start_ns) start_ns[i] = (int64_t)((double)a * 1e6);
    if (end_ns) end_ns[i] = (int64_t)((double)b * 1e6);
  }
}

// ------------------------------------------------------------------------------------------------
// Measured correction: Algorithm 1's `measure latency` on the device
// ------------------------------------------------------------------------------------------------
namespace {
void fill_inputs(const Program& P, cudaStream_t st);
int64_t lower_median(std::vector<double> v);
}  // namespace

Schedule* schedule_measured(const Partition* p, const Profile* pr, const duet_sched_opts* o, const duet_slot* slots,
                            int n_slots, duet_measure_opts* mo) {
  Graph* g = const_cast<Graph*>(p->g);
  auto P = ensure_program(g);
  if (n_slots != pr->n_slots) fail(DUET_EINVAL, "n_slots differs from the profile's slot count");
  duet_measure_opts opts{20, 3, 0, 0};
  if (mo) opts.samples = mo->samples, opts.warmup = mo->warmup;
  if (opts.samples < 1 || opts.warmup < 0) fail(DUET_EINVAL, "bad measure options");
  std::vector<cudaStream_t> streams;
  for (int d = 0; d < n_slots; ++d) {
    if (slots[d].gpu != P->device) fail(DUET_EUNSUPPORTED, "measured mode: every slot must be on the graph's GPU");
    if (!slots[d].stream) fail(DUET_EINVAL, "slot stream is NULL (the legacy default stream cannot be captured)");
    streams.push_back((cudaStream_t)slots[d].stream);
  }
  DeviceGuard dg(P->device);
  cudaStream_t home = streams[0];
  fill_inputs(*P, home);
  for (int s = 0; s < p->n_sg(); ++s) launch_subgraph(*P, *p, s, P->buf, home);  // real data everywhere
  CK(cudaStreamSynchronize(home));
  // Each timed replay starts with a cold L2 (a 256 MB write first, outside the timed interval), as
  // bench.py times every step: a candidate is judged under the condition its latency is reported
  // for (back-to-back warm replays favoured assignments whose inputs stay cached).
  // DUET_MEASURE_FLUSH=0: back-to-back replays.
  static const bool cold = !(getenv("DUET_MEASURE_FLUSH") && atoi(getenv("DUET_MEASURE_FLUSH")) == 0);
  static void* flush_buf = nullptr;
  const size_t flush_bytes = (size_t)256 << 20;
  if (cold && !flush_buf) CK(cudaMalloc(&flush_buf, flush_bytes));
  std::vector<cudaEvent_t> ev(2 * opts.samples + 1);
  for (auto& e : ev) CK(cudaEventCreate(&e));
  std::map<std::vector<int>, int64_t> memo;
  static const bool log = getenv("DUET_MEASURE_LOG") != nullptr;
  const Latency lat = [&](const std::vector<int>& a) -> int64_t {
    auto it = memo.find(a);
    if (it != memo.end()) return it->second;
    auto h0 = std::chrono::steady_clock::now();
    Schedule S;
    S.p = p;
    S.pr = pr;
    S.slot_of = a;
    for (int s = 0; s < p->n_sg(); ++s) S.order.push_back(s);
    int64_t nk = 0;
    ExecEntry E = capture(*P, S, streams, P->buf, {}, {}, &nk);
    auto h1 = std::chrono::steady_clock::now();
    std::vector<double> ns;
    try {
      for (int w = 0; w < opts.warmup; ++w) CK(cudaGraphLaunch(E.exec, home));
      if (cold) {
        for (int k = 0; k < opts.samples; ++k) {
          CK(cudaMemsetAsync(flush_buf, k & 0xff, flush_bytes, home));
          CK(cudaEventRecord(ev[2 * k], home));
          CK(cudaGraphLaunch(E.exec, home));
          CK(cudaEventRecord(ev[2 * k + 1], home));
        }
      } else {
        CK(cudaEventRecord(ev[0], home));
        for (int k = 0; k < opts.samples; ++k) {
          CK(cudaGraphLaunch(E.exec, home));
          CK(cudaEventRecord(ev[k + 1], home));
        }
      }
      CK(cudaStreamSynchronize(home));
      for (int k = 0; k < opts.samples; ++k) {
        float ms = 0;
        if (cold) CK(cudaEventElapsedTime(&ms, ev[2 * k], ev[2 * k + 1]));
        else CK(cudaEventElapsedTime(&ms, ev[k], ev[k + 1]));
        ns.push_back(ms * 1e6);
      }
    } catch (...) {
      cudaGraphExecDestroy(E.exec);
      cudaGraphDestroy(E.graph);
      for (auto e : E.events) cudaEventDestroy(e);
      throw;
    }
    cudaGraphExecDestroy(E.exec);
    cudaGraphDestroy(E.graph);
    for (auto e : E.events) cudaEventDestroy(e);
    int64_t t = lower_median(ns);
    memo[a] = t;
    if (log) {
      auto h2 = std::chrono::steady_clock::now();
      fprintf(stderr, "[measure] #%zu capture+instantiate %.1f ms, timing %.1f ms, latency %lld ns, %lld kernels\n",
              memo.size(), std::chrono::duration<double, std::milli>(h1 - h0).count(),
              std::chrono::duration<double, std::milli>(h2 - h1).count(), (long long)t, (long long)nk);
    }
    return t;
  };
  Schedule* S = nullptr;
  try {
    S = make_schedule_with(p, pr, o, &lat);
  } catch (...) {
    for (auto e : ev) cudaEventDestroy(e);
    throw;
  }
  for (auto e : ev) cudaEventDestroy(e);
  // Final verification against measurement noise (round 2): each candidate above was timed once,
  // at a different moment (clocks drift under the power cap), and Step 3 keeps the minimum of noisy
  // figures.  The K fastest assignments measured (the result included) are timed again, interleaved
  // over R rounds so that drift hits them alike, and the lowest median is kept.  The reported
  // assignment is still one Step 3 evaluated.  DUET_MEASURE_REFINE: K (default 4; <= 1: off).
  static const int refine_k = getenv("DUET_MEASURE_REFINE") ? atoi(getenv("DUET_MEASURE_REFINE")) : 4;
  if (refine_k > 1 && memo.size() > 1 && S->fell_back == 0) {
    std::vector<std::pair<int64_t, std::vector<int>>> ranked;
    for (auto& kv : memo) ranked.push_back({kv.second, kv.first});
    std::sort(ranked.begin(), ranked.end());
    std::vector<std::vector<int>> cands;
    for (size_t i = 0; i < ranked.size() && (int)cands.size() < refine_k; ++i) cands.push_back(ranked[i].second);
    if (std::find(cands.begin(), cands.end(), S->slot_of) == cands.end()) cands.push_back(S->slot_of);
    const int rounds = 6, per = std::max(5, opts.samples / rounds);
    std::vector<ExecEntry> ents;
    std::vector<std::vector<double>> got(cands.size());
    std::vector<cudaEvent_t> e2(2 * per);
    for (auto& e : e2) CK(cudaEventCreate(&e));
    auto cleanup = [&]() {
      for (auto& E : ents) {
        cudaGraphExecDestroy(E.exec);
        cudaGraphDestroy(E.graph);
        for (auto e : E.events) cudaEventDestroy(e);
      }
      for (auto e : e2) cudaEventDestroy(e);
    };
    try {
      for (auto& a : cands) {
        Schedule T;
        T.p = p;
        T.pr = pr;
        T.slot_of = a;
        for (int s = 0; s < p->n_sg(); ++s) T.order.push_back(s);
        int64_t nk = 0;
        ents.push_back(capture(*P, T, streams, P->buf, {}, {}, &nk));
      }
      for (int r = 0; r < rounds; ++r)
        for (size_t c = 0; c < cands.size(); ++c) {
          CK(cudaGraphLaunch(ents[c].exec, home));  // warm the graph, then cold timed replays
          for (int k = 0; k < per; ++k) {
            if (cold) CK(cudaMemsetAsync(flush_buf, k & 0xff, flush_bytes, home));
            CK(cudaEventRecord(e2[2 * k], home));
            CK(cudaGraphLaunch(ents[c].exec, home));
            CK(cudaEventRecord(e2[2 * k + 1], home));
          }
          CK(cudaStreamSynchronize(home));
          for (int k = 0; k < per; ++k) {
            float ms = 0;
            CK(cudaEventElapsedTime(&ms, e2[2 * k], e2[2 * k + 1]));
            got[c].push_back(ms * 1e6);
          }
        }
    } catch (...) {
      cleanup();
      delete S;
      throw;
    }
    cleanup();
    size_t best = 0;
    std::vector<int64_t> med(cands.size());
    for (size_t c = 0; c < cands.size(); ++c) {
      med[c] = lower_median(got[c]);
      if (med[c] < med[best]) best = c;
    }
    if (log)
      for (size_t c = 0; c < cands.size(); ++c)
        fprintf(stderr, "[refine] candidate %zu first %lld ns, interleaved %lld ns%s\n", c,
                (long long)memo[cands[c]], (long long)med[c], c == best ? " (kept)" : "");
    S->slot_of = cands[best];
    S->measured_ns = med[best];
  }
  if (mo) {
    mo->measured_ns = S->measured_ns;
    mo->evaluations = (int32_t)memo.size();
  }
  return S;
}

int64_t schedule_launch_count(const Schedule* s) {
  if (!s->exec) fail(DUET_ESTATE, "launch count is known after the first duet_run");
  return s->exec->launches;
}

void node_run(Graph* g, const std::string& name, const duet_tensor* args, int n_args, duet_tensor* out, void* stream) {
  auto it = g->by_name.find(name);
  if (it == g->by_name.end()) fail(DUET_EINVAL, "no node %" + name);
  const Node& nd = g->nodes[it->second];
  auto P = ensure_program(g);
  if (n_args != (int)nd.arg_nodes.size()) fail(DUET_EINVAL, "node_run: wrong number of arguments");
  DeviceGuard dg(P->device);
  Ptrs T = P->buf;
  for (int i = 0; i < n_args; ++i) {
    const Node& a = g->nodes[nd.arg_nodes[i]];
    check_tensor(a, args[i], "argument");
    if (args[i].device != P->device) fail(DUET_EINVAL, "node_run: arguments must be device tensors on the graph's GPU");
    T[a.id] = args[i].data;
  }
  check_tensor(nd, *out, "output");
  if (out->device != P->device) fail(DUET_EINVAL, "node_run: output must be a device tensor");
  T[nd.id] = out->data;
  if (!P->ops[nd.id].launch) fail(DUET_EINVAL, "node %" + name + " has no kernel");
  P->ops[nd.id].launch(T, (cudaStream_t)stream);
}

// ------------------------------------------------------------------------------------------------
// Profiler
// ------------------------------------------------------------------------------------------------
namespace {

__global__ void tiny_kernel(int* p) {
  if (threadIdx.x == 0 && p) atomicAdd(p, 1);
}

// Synthetic but representative data in the input staging buffers: uniformly distributed ids so
// gathers touch the whole table (zeros would hit one cached row), N(0,1)-scaled floats.
void fill_inputs(const Program& P, cudaStream_t st) {
  const Graph& g = *P.g;
  for (int id : g.input_nodes) {
    const Node& n = g.nodes[id];
    int64_t high = 0;
    for (auto& c : g.nodes)
      for (size_t k = 0; k < c.arg_nodes.size(); ++k)
        if (c.arg_nodes[k] == id && c.op == "embed_seq") high = g.params.at(c.params[0]).shape[0];
    if (n.dtype == kI32 && high == 0) high = 1;
    fill_random(P.buf[id], n.dtype, n.numel(), high, 0x5EED + id, st);
  }
}

int64_t lower_median(std::vector<double> v) {
  std::sort(v.begin(), v.end());
  double m = v[(v.size() - 1) / 2];
  return (int64_t)(m + 0.5);
}

}  // namespace

Profile* profile_on_device(const Partition* p, const duet_slot* slots, int n_slots, const duet_profile_opts* o) {
  Graph* g = const_cast<Graph*>(p->g);
  auto P = ensure_program(g);
  duet_profile_opts opts{20, 500, 20, 0};
  if (o) opts = *o;
  if (opts.samples < 1 || opts.reps_per_sample < 1 || opts.warmup < 0) fail(DUET_EINVAL, "bad profile options");
  for (int d = 0; d < n_slots; ++d)
    if (slots[d].gpu != P->device) fail(DUET_EUNSUPPORTED, "profiling slots on another GPU is not supported");
  DeviceGuard dg(P->device);
  cudaStream_t st;
  CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  std::unique_ptr<Profile> pr(new Profile());
  pr->p = p;
  pr->n_slots = n_slots;
  for (int d = 0; d < n_slots; ++d) pr->slot_gpu.push_back(slots[d].gpu);
  const int n = p->n_sg();
  pr->t_ns.assign((size_t)n * n_slots, 0);
  std::vector<cudaEvent_t> ev(opts.samples + 1);
  try {
    for (auto& e : ev) CK(cudaEventCreate(&e));
    fill_inputs(*P, st);
    // one serial pass so every intermediate buffer holds real data
    for (int s = 0; s < n; ++s) launch_subgraph(*P, *p, s, P->buf, st);
    CK(cudaStreamSynchronize(st));
    for (int s = 0; s < n; ++s) {
      cudaGraph_t gr;
      cudaGraphExec_t ex;
      // R back-to-back copies of the subgraph inside ONE graph: a sample is one graph launch, so
      // the per-launch overhead of cudaGraphLaunch is amortised over R subgraph executions.
      CK(cudaStreamBeginCapture(st, cudaStreamCaptureModeRelaxed));
      for (int r = 0; r < opts.reps_per_sample; ++r) launch_subgraph(*P, *p, s, P->buf, st);
      CK(cudaStreamEndCapture(st, &gr));
      CK(cudaGraphInstantiate(&ex, gr, 0));
      for (int w = 0; w < std::max(1, opts.warmup / std::max(1, opts.reps_per_sample)) + 1; ++w) CK(cudaGraphLaunch(ex, st));
      CK(cudaEventRecord(ev[0], st));
      for (int k = 0; k < opts.samples; ++k) {
        CK(cudaGraphLaunch(ex, st));
        CK(cudaEventRecord(ev[k + 1], st));
      }
      CK(cudaStreamSynchronize(st));
      std::vector<double> ns;
      for (int k = 0; k < opts.samples; ++k) {
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, ev[k], ev[k + 1]));
        ns.push_back(ms * 1e6 / opts.reps_per_sample);
      }
      int64_t t = lower_median(ns);
      for (int d = 0; d < n_slots; ++d) pr->t_ns[(size_t)s * n_slots + d] = t;
      cudaGraphExecDestroy(ex);
      cudaGraphDestroy(gr);
    }
    if (opts.calibrate_comm && n_slots > 1) {
      // alpha_same = extra latency of a cross-stream dependency inside a graph (Fig. 5)
      cudaStream_t s2;
      CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
      cudaEvent_t e1, e2;
      CK(cudaEventCreateWithFlags(&e1, cudaEventDisableTiming));
      CK(cudaEventCreateWithFlags(&e2, cudaEventDisableTiming));
      auto time_graph = [&](bool cross) {
        cudaGraph_t gr;
        cudaGraphExec_t ex;
        CK(cudaStreamBeginCapture(st, cudaStreamCaptureModeRelaxed));
        for (int i = 0; i < 8; ++i) {
          if (cross) {
            CK(cudaEventRecord(e1, st));
            CK(cudaStreamWaitEvent(s2, e1, 0));
            tiny_kernel<<<1, 32, 0, s2>>>(nullptr);
            CK(cudaEventRecord(e2, s2));
            CK(cudaStreamWaitEvent(st, e2, 0));
          } else {
            tiny_kernel<<<1, 32, 0, st>>>(nullptr);
          }
          tiny_kernel<<<1, 32, 0, st>>>(nullptr);
        }
        CK(cudaStreamEndCapture(st, &gr));
        CK(cudaGraphInstantiate(&ex, gr, 0));
        for (int w = 0; w < 20; ++w) CK(cudaGraphLaunch(ex, st));
        CK(cudaEventRecord(ev[0], st));
        for (int k = 0; k < 200; ++k) CK(cudaGraphLaunch(ex, st));
        CK(cudaEventRecord(ev[1], st));
        CK(cudaStreamSynchronize(st));
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, ev[0], ev[1]));
        cudaGraphExecDestroy(ex);
        cudaGraphDestroy(gr);
        return ms * 1e6 / 200.0 / 16.0;  // per dependency edge (2 edges per iteration)
      };
      double same = time_graph(false), cross = time_graph(true);
      pr->comm.same_gpu.alpha_ns = std::max<int64_t>(0, (int64_t)((cross - same) + 0.5));
      cudaEventDestroy(e1);
      cudaEventDestroy(e2);
      cudaStreamDestroy(s2);
    }
  } catch (...) {
    for (auto e : ev)
      if (e) cudaEventDestroy(e);
    cudaStreamDestroy(st);
    throw;
  }
  for (auto e : ev) cudaEventDestroy(e);
  CK(cudaStreamDestroy(st));
  return pr.release();
}

}  // namespace duet
