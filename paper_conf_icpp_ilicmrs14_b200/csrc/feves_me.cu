// feves_me.cu -- libfeves_me.so: the C-ABI of include/feves_me.h over the
// sm_100a kernels (me_fsbm.cuh, int_subpel.cuh, sme_refine.cuh).
//
// The context owns: the spiral-rank tables of G4 (built here with the CLOSED
// FORM; the oracle enumerates the spiral independently), ME scratch for
// me_encode_frame, and its stream.  No allocation on the per-frame path.
#include "../../include/feves_me.h"

#include <cuda.h>   // CUdeviceptr / CUresult types only: driver calls go through cudaGetDriverEntryPoint

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <algorithm>
#include <mutex>
#include <vector>

#include "int_subpel.cuh"
#include "launch.cuh"   // ME / SME launches (their own translation units: me_s*.cu, sme.cu)
#include "sme_smem.cuh"  // kSme2Mb (staged SME group size)
#include "mode_decision.cuh"

using namespace feves;

struct me_ctx {
  int W, H, S, R, n_rf;
  int mb_cols, mb_rows, row0, row1;
  int sf_pad, sf_pitch, sf_rows;
  int device;
  cudaStream_t stream;
  cudaStream_t own;      // the context's own stream (created in me_create, destroyed in me_destroy)
  uint32_t* d_rank;      // [S][Sp]: [dx+R][dy+R], column pitch Sp = S rounded up to 4 (me_rank_pitch)
  uint32_t* d_inv;       // [(S+1)^2]
  uint32_t* d_glob;      // [4][4096]: S = 128 quadrant-local rank -> global dense rank
  int16_t* d_mvs;        // scratch for me_encode_frame (full frame)
  uint16_t* d_sads;
  // ME launch geometry
  int me_threads;
  size_t me_smem;
  int last_launches;
  // IPPP stream state (me_stream_push): ring of n_rf+1 frames, n_rf SFs
  uint8_t* ring;         // (n_rf+1) * W*H
  uint8_t* sf_ring;      // n_rf * 16*sf_rows*sf_pitch
  int16_t* d_qmvs;       // device outputs of the last push
  uint16_t* d_qsads;
  long long t;           // frames pushed since reset
  cudaStream_t side;     // INT runs here, concurrently with ME
  cudaEvent_t ev_fork, ev_join;
  // host-buffer pushes: uploads / downloads on their own streams so the copy engines
  // overlap the compute of the neighbouring frames (P:51 copy engines, Fig. 4 VCM)
  cudaStream_t copy_in, copy_out;
  cudaEvent_t ev_done[2];     // compute of push t finished (ring: t & 1)
  cudaEvent_t ev_up[2];       // upload of push t finished
  cudaEvent_t ev_down[2];     // download of push t finished (frees device output buffer t & 1)
  int16_t* d_qmvs2[2];        // double-buffered device outputs for host pushes
  uint16_t* d_qsads2[2];
  // per-module timers ("facilities to measure execution ... times")
  int timing;
  cudaEvent_t ev_t[6];   // INT start/stop (side stream), ME start/stop, SME start/stop
  int timed_mask;        // which pairs were recorded by the last push/encode
  int fuse;              // run SME inside the ME kernel (ME_OPT_FUSED_SME)
  size_t me_smem_fused;
  int pipeline;          // per-RF ME launches, SME of RF k co-running with ME of RF k+1 (ME_OPT_PIPELINE_RF)
  int me_ctas_per_sm;    // cap on resident ME CTAs per SM (0 = hardware maximum; ME_OPT_ME_CTAS_PER_SM)
  int lambda;            // G18 rate term (ME_OPT_LAMBDA); key = J * kmul + rank
  int satd;              // G20 SME distortion = Hadamard SATD (ME_OPT_SME_SATD)
  int inclusive;         // G1 alternative: candidates [-R, R]^2 (ME_OPT_SA_INCLUSIVE)
  int max_pmv;           // G21: predictor clamp (me_create_pmv); > 0 routes ME to the runtime-S kernel
  const int16_t* d_pmv;  // G21: predictor field (me_set_pmv), device, or null = zero predictor
  uint32_t kmul;
  int kshift;
  cudaStream_t sme_st;   // pipeline: SME stream
  cudaEvent_t ev_me[kMaxRf], ev_sme_done;
  int sf_v0[kMaxRf], sf_v1[kMaxRf];   // MB rows whose SF rows each SF-ring slot holds (re-split support)
  int halo_only;                      // ME_OPT_HALO_ONLY: pushes copy the stripe + halo rows only
  int overlap;                        // ME_OPT_OVERLAP_SME: SME(t) on its own stream, co-running with ME(t+1)
  cudaStream_t ov_st;                 // overlap: SME stream (high priority)
  cudaEvent_t ev_ov_me, ev_ov_sme;    // overlap: ME(t) done, SME(t) done
  int16_t* d_mvs_ov[2];               // overlap: ME outputs double-buffered (SME(t) reads while ME(t+1) writes)
  uint16_t* d_sads_ov[2];
  bool ov_pending;                    // an SME of an earlier push may still run on ov_st
  int fv0[kMaxRf + 2], fv1[kMaxRf + 2];   // frame rows each frame-ring slot holds
  struct Peer { uintptr_t lo, hi; void* base; } peers[16];   // me_ipc_open mappings
  int n_peers;
  cudaEvent_t ev_switch;   // me_set_stream: orders the old stream's work before the new one's
  // ME_OPT_GRAPH: one captured CUDA graph per ring phase of the device-resident stream
  struct Graph {
    cudaGraphExec_t exec;
    cudaGraph_t graph;     // kept: its frame-copy node is re-pointed at each replay's frame
    cudaGraphNode_t copy;  // the frame's D2D copy into the ring slot
    const void* cf; const void* qm; const void* qs;
    int row0, row1;
    long long epoch;
    int timing, launches, timed_mask;
  };
  std::vector<Graph> graphs;
  int graph;             // ME_OPT_GRAPH
  int sme_kernel;        // ME_OPT_SME_KERNEL: 0 global-load SME (default), 1 shared-memory staged
  int int_kernel;        // ME_OPT_INT_KERNEL: 0 per-thread global loads, 1 shared-memory tiled
  int rf_per_cta;        // ME_OPT_RF_PER_CTA: RFs per ME CTA (0 = all, -1 = auto)
  int sme_split;         // ME_OPT_SME_SPLIT: 0 auto, 1 never, 2 always (one partition group per SME warp)
  int sme_split_warps;   // auto: split below this many mode-warps
  // me_stream_push_flags: stream-ordered peer flags of the push being enqueued
  const uint32_t* wait_flag; uint32_t wait_value;     // the frame copy waits for *wait_flag >= wait_value
  uint32_t* signal_flag; uint32_t signal_value;       // written once the push's outputs are complete
  int* d_ovf;            // staged SME overflow list: [0] count, then (MB, RF) items
  bool capturing;        // push_enqueue runs inside a stream capture
  long long gepoch;      // bumped by every setting change: cached graphs are stale
};

static thread_local int g_last_error = ME_OK;
constexpr int kNPhase = 16;

// ------------------------------------------------------------- helpers ----
static int spiral_rank_closed_form(int dx, int dy) {   // G4
  const int l = std::max(std::abs(dx), std::abs(dy));
  if (l == 0) return 0;
  const int base = (2 * l - 1) * (2 * l - 1);
  if (std::abs(dy) == l && std::abs(dx) < l) return base + 2 * (dx + l - 1) + (dy > 0 ? 1 : 0);
  return base + 2 * (2 * l - 1) + 2 * (dy + l) + (dx > 0 ? 1 : 0);
}

static bool is_peer_ptr(const me_ctx* c, const void* p) {
  for (int i = 0; i < c->n_peers; ++i)
    if (c->peers[i].base && reinterpret_cast<uintptr_t>(p) >= c->peers[i].lo &&
        reinterpret_cast<uintptr_t>(p) < c->peers[i].hi)
      return true;
  return false;
}

// checked on every call (no cache: a freed and re-allocated range must be re-checked)
static bool is_device_ptr(me_ctx* c, const void* p) {
  if (!p) return false;
  if (is_peer_ptr(c, p)) return true;   // peer memory mapped by me_ipc_open (another GPU's buffer)
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) { cudaGetLastError(); return false; }
  return (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) && a.device == c->device;
}

static cudaError_t set_me_smem(int bytes) {
  cudaError_t e = me_set_smem_0(bytes);
  if (e == cudaSuccess) e = me_set_smem_16(bytes);
  if (e == cudaSuccess) e = me_set_smem_32(bytes);
  if (e == cudaSuccess) e = me_set_smem_64(bytes);
  if (e == cudaSuccess) e = me_set_smem_128(bytes);
  return e;
}

static void graphs_drop(me_ctx* c) {
  for (auto& g : c->graphs) {
    if (g.exec) cudaGraphExecDestroy(g.exec);
    if (g.graph) cudaGraphDestroy(g.graph);
  }
  c->graphs.clear();
}

// Stream memory operations (driver API, through cudaGetDriverEntryPoint like alloc_base):
// a stream waits until a 32-bit device word (local or a peer's, me_ipc_open) is >= value, or
// writes one after its preceding work -- the stream-ordered flags of the multi-GPU exchange.
using StreamValueFn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
static StreamValueFn driver_fn(const char* name) {
  void* f = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &f, cudaEnableDefault, &q) != cudaSuccess || !f || q != cudaDriverEntryPointSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return reinterpret_cast<StreamValueFn>(f);
}
static int stream_wait_value(cudaStream_t s, const uint32_t* flag, uint32_t value) {
  static StreamValueFn fn = driver_fn("cuStreamWaitValue32");
  if (!fn) return ME_ECUDA;
  return fn(reinterpret_cast<CUstream>(s), reinterpret_cast<CUdeviceptr>(flag), value, CU_STREAM_WAIT_VALUE_GEQ) ==
                 CUDA_SUCCESS
             ? ME_OK
             : ME_ECUDA;
}
static int stream_write_value(cudaStream_t s, uint32_t* flag, uint32_t value) {
  static StreamValueFn fn = driver_fn("cuStreamWriteValue32");
  if (!fn) return ME_ECUDA;
  return fn(reinterpret_cast<CUstream>(s), reinterpret_cast<CUdeviceptr>(flag), value, CU_STREAM_WRITE_VALUE_DEFAULT) ==
                 CUDA_SUCCESS
             ? ME_OK
             : ME_ECUDA;
}

static int launch_status() {
  const cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) { fprintf(stderr, "feves_me: %s\n", cudaGetErrorString(e)); return ME_ECUDA; }
  return ME_OK;
}

// key addend table E[dy+R][dx+R] = lambda * R(4dx, 4dy) * kmul + spiral rank (G4, G18):
// with lambda = 0 this is the spiral rank and key = SAD * 2^16 + rank; with a rate
// term J = SAD + lambda*R may exceed 16 bits, so key = J * 2^15 + rank (rank < 2^15
// for S <= 128).  The key is 32 bits, so J must stay below 2^17: with the 16x16 SAD
// up to 65280 that caps lambda at (2^17 - 1 - 65280) / max R over the SA offsets
// (lambda_limit: 1935 at S = 64, 1731 at S = 128; the API's own cap is 2000).
static int lambda_limit(int S, int inclusive) {
  const int R = S / 2, hi = S + inclusive - 1 - R;
  int rmax = 0;
  for (int d = -R; d <= hi; ++d) rmax = std::max(rmax, se_bits(4 * d));
  return std::min(2000, ((1 << 17) - 1 - 65280) / (2 * rmax));
}

// Host-only construction of the three ME key tables (no CUDA call; me_key_tables exposes it).
// e: [Sc][Sp] key addends, [dx+R][dy+R]; inv: dense rank -> packed MV; glob: S = 128 quadrant map.
static void build_key_tables(int S, int inclusive, int lambda, std::vector<uint32_t>& e, std::vector<uint32_t>& inv,
                             std::vector<uint32_t>& glob, bool allow_quad = true) {
  const int R = S / 2, Sc = S + inclusive, hi = Sc - 1 - R;   // candidates per axis, dx,dy in [-R, hi]
  const uint32_t kmul = 1u << (lambda ? 15 : 16);
  const int Sp = me_rank_pitch(Sc);
  e.assign((size_t)Sc * Sp, 0);
  inv.assign((size_t)(S + 1) * (S + 1), 0);
  glob.assign(4 * 4096, 0);
  // DENSE rank: the candidates of the SA numbered 0..Sc^2-1 in spiral order (G4).  It
  // orders candidates exactly as the spiral rank does, and < 4096 for S <= 64 is what
  // lets the ME kernel build parent keys as sums of child keys (me_fsbm.cuh, SumKeys).
  std::vector<std::pair<int, uint32_t>> order;
  order.reserve((size_t)Sc * Sc);
  for (int dy = -R; dy <= hi; ++dy)
    for (int dx = -R; dx <= hi; ++dx)
      order.emplace_back(spiral_rank_closed_form(dx, dy), (uint32_t)(uint16_t)dx | ((uint32_t)(uint16_t)dy << 16));
  std::sort(order.begin(), order.end());
  // S = 128, pure SAD: the ME kernel sums keys quadrant by quadrant (me_fsbm.cuh QuadKeys),
  // so its table holds the rank inside the candidate's quadrant, and glob maps it back
  const bool quad = S == 128 && !inclusive && !lambda && allow_quad;
  int qn[4] = {0, 0, 0, 0};
  for (size_t r = 0; r < order.size(); ++r) {
    const int dx = (int)(int16_t)(order[r].second & 0xffffu), dy = (int)(int16_t)(order[r].second >> 16);
    uint32_t key_rank = (uint32_t)r;
    if (quad) {
      const int q = 2 * (dy >= 0) + (dx >= 0);
      glob[q * 4096 + qn[q]] = (uint32_t)r;
      key_rank = (uint32_t)qn[q]++;
    }
    e[(size_t)(dx + R) * Sp + (dy + R)] = (uint32_t)(lambda * (se_bits(4 * dx) + se_bits(4 * dy))) * kmul + key_rank;
    inv[r] = order[r].second;
  }
}

extern "C" int me_key_tables(int sa_range, int inclusive, int lambda, uint32_t* key_addend, uint32_t* inv,
                             uint32_t* glob) {
  if (sa_range < 4 || sa_range > 128 || (sa_range & 1) || (inclusive != 0 && inclusive != 1) || lambda < 0 ||
      lambda > lambda_limit(sa_range, inclusive) || !key_addend || !inv || !glob)
    return ME_EINVAL;
  std::vector<uint32_t> e, iv, g;
  build_key_tables(sa_range, inclusive, lambda, e, iv, g);
  std::copy(e.begin(), e.end(), key_addend);
  std::copy(iv.begin(), iv.end(), inv);
  std::copy(g.begin(), g.end(), glob);
  return ME_OK;
}

static int upload_key_table(me_ctx* c) {
  const int Sc = c->S + c->inclusive;
  c->kshift = c->lambda ? 15 : 16;
  c->kmul = 1u << c->kshift;
  std::vector<uint32_t> e, inv, glob;
  build_key_tables(c->S, c->inclusive, c->lambda, e, inv, glob, c->max_pmv == 0);
  c->me_threads = me_threads(Sc);
  c->me_smem = (size_t)me_smem_words(Sc) * 4;
  c->me_smem_fused = (size_t)me_smem_words_fused(Sc, c->n_rf) * 4;
  return cudaMemcpy(c->d_rank, e.data(), e.size() * 4, cudaMemcpyHostToDevice) == cudaSuccess &&
                 cudaMemcpy(c->d_inv, inv.data(), inv.size() * 4, cudaMemcpyHostToDevice) == cudaSuccess &&
                 cudaMemcpy(c->d_glob, glob.data(), glob.size() * 4, cudaMemcpyHostToDevice) == cudaSuccess
             ? ME_OK
             : ME_ECUDA;
}

// ------------------------------------------------------------ lifetime ----
// The context's own stream runs at the highest priority and the INT side stream at the
// lowest: INT (concurrent with ME) then only takes SMs that ME's CTAs leave free, i.e. it
// fills ME's last-wave tail instead of delaying ME's first wave.  Stream-captured graphs keep
// these as per-node priorities (cudaGraphInstantiateFlagUseNodePriority).
static cudaError_t create_own_stream(me_ctx* c) {
  int least = 0, greatest = 0;
  cudaDeviceGetStreamPriorityRange(&least, &greatest);
  return cudaStreamCreateWithPriority(&c->own, cudaStreamNonBlocking, greatest);
}

extern "C" me_ctx* me_create(int width, int height, int sa_range, int n_rf) {
  return me_create_pmv(width, height, sa_range, n_rf, 0);
}

extern "C" me_ctx* me_create_pmv(int width, int height, int sa_range, int n_rf, int max_pmv) {
  g_last_error = ME_EINVAL;
  if (width <= 0 || height <= 0 || width > 16384 || height > 16384) return nullptr;
  if (sa_range < 4 || sa_range > 128 || (sa_range & 1)) return nullptr;
  if (max_pmv < 0 || max_pmv > 256 || (max_pmv > 0 && sa_range == 128)) return nullptr;
  if (n_rf < 1 || n_rf > kMaxRf) return nullptr;
  me_ctx* c = new (std::nothrow) me_ctx();
  if (!c) { g_last_error = ME_ENOMEM; return nullptr; }
  c->W = width; c->H = height; c->S = sa_range; c->R = sa_range / 2; c->n_rf = n_rf;
  c->mb_cols = (width + 15) / 16; c->mb_rows = (height + 15) / 16;
  c->row0 = 0; c->row1 = c->mb_rows;
  c->max_pmv = max_pmv;   // G21: every MV stays within p +- R, |p| <= max_pmv -> SF margin covers it
  c->sf_pad = ((c->R + max_pmv + 4 + 15) / 16) * 16;
  c->sf_pitch = 16 * c->mb_cols + 2 * c->sf_pad;
  c->sf_rows = 16 * c->mb_rows + 2 * c->sf_pad;
  if (cudaGetDevice(&c->device) != cudaSuccess) { delete c; g_last_error = ME_ECUDA; return nullptr; }

  // lane geometry (me_fsbm.cuh): 32 dx per warp (fewer lanes per dx group for
  // small SAs, the rest of the warp takes other dy sub-ranges)
  const int S = c->S;
  c->me_threads = me_threads(S);
  c->me_smem = (size_t)me_smem_words(S) * 4;
  c->me_smem_fused = (size_t)me_smem_words_fused(S, n_rf) * 4;
  c->fuse = 0;   // measured slower on B200: opt-in
  c->pipeline = 0;
  c->me_ctas_per_sm = 0;

  const size_t nmv = (size_t)c->mb_cols * c->mb_rows * n_rf * kNPart;
  bool ok = cudaMalloc(&c->d_rank, (size_t)(S + 1) * me_rank_pitch(S + 1) * 4) == cudaSuccess &&
            cudaMalloc(&c->d_inv, (size_t)(S + 1) * (S + 1) * 4) == cudaSuccess &&
            cudaMalloc(&c->d_glob, (size_t)4 * 4096 * 4) == cudaSuccess &&
            cudaMalloc(&c->d_mvs, nmv * 4) == cudaSuccess &&
            cudaMalloc(&c->d_sads, nmv * 2) == cudaSuccess &&
            cudaMalloc(&c->d_ovf, (1 + (size_t)c->mb_cols * c->mb_rows * n_rf) * sizeof(int)) == cudaSuccess &&
            create_own_stream(c) == cudaSuccess;
  if (ok) {
    c->stream = c->own;
    c->int_kernel = 1;   // shared-memory tiled INT: 11.2 vs 14.2 us (ncu, 1080p S64)
    c->sme_split = 0;
    int sms = 148;
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, c->device) != cudaSuccess) sms = 148;
    c->sme_split_warps = 6 * sms * 20;   // ~ six waves of the SME kernel (20 resident warps/SM): 1080p on 2+ GPUs
    c->rf_per_cta = -1;  // auto: one CTA per (MB, RF) (1080p S64 4 RF ME 818.5 vs 834.5 us, 9-row stripe
                         // 124.1 vs 144.8 us); 2 RFs per CTA at S = 128 (2160p ME 12.50 vs 12.62 ms)
    c->sme_kernel = 0;   // the staged SME measured on par (145-149 vs 145 us at 1080p S64 4 RF): opt-in
    ok = upload_key_table(c) == ME_OK && sme2_init() == cudaSuccess &&
         set_me_smem(200 * 1024) == cudaSuccess;   // max; the launch asks for what it needs
  }
  if (!ok) {
    cudaGetLastError();
    me_destroy(c);
    g_last_error = ME_ENOMEM;
    return nullptr;
  }
  g_last_error = ME_OK;
  return c;
}

extern "C" void me_destroy(me_ctx* c) {
  if (!c) return;
  if (c->stream) cudaStreamSynchronize(c->stream);
  if (c->own) cudaStreamSynchronize(c->own);
  if (c->copy_in) cudaStreamSynchronize(c->copy_in);
  if (c->copy_out) cudaStreamSynchronize(c->copy_out);
  if (c->side) cudaStreamSynchronize(c->side);
  if (c->sme_st) cudaStreamSynchronize(c->sme_st);
  cudaFree(c->d_rank);
  cudaFree(c->d_inv);
  cudaFree(c->d_glob);
  cudaFree(c->d_mvs);
  cudaFree(c->d_sads);
  cudaFree(c->d_ovf);
  cudaFree(c->ring);
  cudaFree(c->sf_ring);
  cudaFree(c->d_qmvs);
  cudaFree(c->d_qsads);
  for (int i = 0; i < 6; ++i)
    if (c->ev_t[i]) cudaEventDestroy(c->ev_t[i]);
  for (int i = 0; i < 2; ++i) {
    if (c->ev_done[i]) cudaEventDestroy(c->ev_done[i]);
    if (c->ev_up[i]) cudaEventDestroy(c->ev_up[i]);
    if (c->ev_down[i]) cudaEventDestroy(c->ev_down[i]);
    cudaFree(c->d_qmvs2[i]);
    cudaFree(c->d_qsads2[i]);
  }
  for (int i = 0; i < kMaxRf; ++i)
    if (c->ev_me[i]) cudaEventDestroy(c->ev_me[i]);
  if (c->ev_sme_done) cudaEventDestroy(c->ev_sme_done);
  if (c->sme_st) cudaStreamDestroy(c->sme_st);
  if (c->copy_in) cudaStreamDestroy(c->copy_in);
  if (c->copy_out) cudaStreamDestroy(c->copy_out);
  if (c->side) cudaStreamDestroy(c->side);
  if (c->ev_fork) cudaEventDestroy(c->ev_fork);
  if (c->ev_join) cudaEventDestroy(c->ev_join);
  if (c->ev_switch) cudaEventDestroy(c->ev_switch);
  graphs_drop(c);
  if (c->own) cudaStreamDestroy(c->own);
  for (int i = 0; i < c->n_peers; ++i)
    if (c->peers[i].base) cudaIpcCloseMemHandle(c->peers[i].base);
  if (c->ov_st) { cudaStreamSynchronize(c->ov_st); cudaStreamDestroy(c->ov_st); }
  if (c->ev_ov_me) cudaEventDestroy(c->ev_ov_me);
  if (c->ev_ov_sme) cudaEventDestroy(c->ev_ov_sme);
  for (int i = 0; i < 2; ++i) { cudaFree(c->d_mvs_ov[i]); cudaFree(c->d_sads_ov[i]); }
  delete c;
}

extern "C" int me_last_error(void) { return g_last_error; }

extern "C" const char* me_strerror(int s) {
  switch (s) {
    case ME_OK: return "ok";
    case ME_EINVAL: return "invalid argument";
    case ME_ENOMEM: return "out of memory";
    case ME_ECUDA: return "CUDA error";
    case ME_ESTATE: return "bad context state";
    default: return "unknown status";
  }
}

// ME_STREAM_OWN = the context's own stream again (it lives until me_destroy).  Work
// already enqueued on the previous stream is ordered before later work by an event
// (no host synchronisation).
extern "C" int me_set_stream(me_ctx* c, void* s) {
  if (!c) return ME_EINVAL;
  cudaStream_t ns = s == ME_STREAM_OWN ? c->own : (cudaStream_t)s;
  if (ns == c->stream) return ME_OK;
  if (!c->ev_switch && cudaEventCreateWithFlags(&c->ev_switch, cudaEventDisableTiming) != cudaSuccess)
    return launch_status();
  if (cudaEventRecord(c->ev_switch, c->stream) != cudaSuccess || cudaStreamWaitEvent(ns, c->ev_switch, 0) != cudaSuccess)
    return launch_status();
  c->stream = ns;
  c->gepoch++;
  return ME_OK;
}

extern "C" int me_set_rows(me_ctx* c, int r0, int r1) {
  if (!c || r0 < 0 || r1 > c->mb_rows || r0 >= r1) return ME_EINVAL;
  c->row0 = r0; c->row1 = r1;
  c->gepoch++;
  return ME_OK;
}

extern "C" int me_get_layout(const me_ctx* c, int* mb_cols, int* mb_rows, int* sf_pad, int* sf_pitch,
                             int* sf_rows) {
  if (!c) return ME_EINVAL;
  if (mb_cols) *mb_cols = c->mb_cols;
  if (mb_rows) *mb_rows = c->mb_rows;
  if (sf_pad) *sf_pad = c->sf_pad;
  if (sf_pitch) *sf_pitch = c->sf_pitch;
  if (sf_rows) *sf_rows = c->sf_rows;
  return ME_OK;
}

extern "C" int me_last_launch_count(const me_ctx* c) { return c ? c->last_launches : -1; }

// --------------------------------------------------------------- launches ----
static void tmark(me_ctx* c, int i, cudaStream_t st) {
  if (!c->timing) return;
  if (c->capturing) cudaEventRecordWithFlags(c->ev_t[i], st, cudaEventRecordExternal);   // a graph node
  else cudaEventRecord(c->ev_t[i], st);
  c->timed_mask |= 1 << (i / 2);
}

// ME (and, when sfs != NULL, the fused SME of me_fsbm.cuh) over n_ref RFs
static int launch_me(me_ctx* c, const uint8_t* cf, const uint8_t* const* rfs, int16_t* mvs, uint16_t* sads,
                     int n_ref, cudaStream_t st, const uint8_t* const* sfs = nullptr, int16_t* qmvs = nullptr,
                     uint16_t* qsads = nullptr, int rf0 = 0) {
  if (n_ref <= 0) return ME_OK;   // nothing to search (the kernel would write nothing)
  MeParams P;
  memset(&P, 0, sizeof(P));
  P.cf = cf;
  for (int k = 0; k < n_ref; ++k) P.rf[k] = rfs[k];
  P.W = c->W; P.H = c->H; P.S = c->S + c->inclusive; P.R = c->R; P.n_rf = n_ref; P.rf_stride = c->n_rf;
  P.mb_cols = c->mb_cols; P.row0 = c->row0;
  P.rank_tab = c->d_rank; P.inv_tab = c->d_inv; P.glob_tab = c->d_glob;
  P.kmul = c->kmul; P.kshift = c->kshift; P.lambda = c->lambda;
  P.out_mvs = mvs; P.out_sads = sads;
  P.pmv = c->d_pmv ? c->d_pmv + 2 * rf0 : nullptr;   // rf0: first RF of this launch (per-RF pipeline)
  P.max_pmv = c->max_pmv;
  bool vec = (c->W % 16 == 0) && (c->R % 16 == 0);
  for (int k = 0; k < n_ref; ++k) vec = vec && ((reinterpret_cast<uintptr_t>(rfs[k]) & 15) == 0);
  P.vec_ok = vec ? 1 : 0;
  const bool fused = sfs != nullptr;
  if (fused) {
    for (int k = 0; k < n_ref; ++k) P.sf[k] = sfs[k];
    P.sf_pad = c->sf_pad; P.sf_pitch = c->sf_pitch;
    P.sf_plane = (size_t)c->sf_rows * c->sf_pitch;
    P.out_qmvs = reinterpret_cast<uint32_t*>(qmvs);
    P.out_qsads = qsads;
  }
  // RFs per CTA (ME_OPT_RF_PER_CTA, default 1: one CTA per (MB, RF)): more, shorter CTAs
  // desynchronise their window stagings across waves and shorten the last wave -- the frame and,
  // more so, a narrow MB-row stripe of a multi-GPU split
  int rpc = std::max(1, n_ref);
  const int want = c->rf_per_cta < 0 ? (c->S >= 128 ? 2 : 1) : c->rf_per_cta;
  if (!fused && want > 0) rpc = std::max(1, std::min(n_ref, want));
  P.rf_per_cta = rpc;
  dim3 grid(c->mb_cols, c->row1 - c->row0, (n_ref + rpc - 1) / rpc);
  size_t smem = fused ? c->me_smem_fused : c->me_smem;
  if (c->me_ctas_per_sm > 0)   // occupancy cap: leave registers / warps for a co-running SME
    smem = std::max(smem, (size_t)(228 * 1024) / (size_t)(c->me_ctas_per_sm + 1) - 1024 + 64);
  tmark(c, 2, st);
  const int variant = fused ? kMeFused
                    : c->max_pmv ? (c->lambda ? kMePmvRate : kMePmv)
                    : c->lambda ? kMeRate : kMePlain;
  cudaError_t e;
  switch (c->inclusive || (c->max_pmv && c->S == 128) ? 0 : c->S) {   // compile-time window geometry for the paper's SA sizes (Fig. 6a: 32..256)
    case 16: e = me_launch_16(variant, grid, c->me_threads, smem, st, P); break;
    case 32: e = me_launch_32(variant, grid, c->me_threads, smem, st, P); break;
    case 64: e = me_launch_64(variant, grid, c->me_threads, smem, st, P); break;
    case 128: e = me_launch_128(variant, grid, c->me_threads, smem, st, P); break;
    default: e = me_launch_0(variant, grid, c->me_threads, smem, st, P); break;
  }
  if (e != cudaSuccess) { fprintf(stderr, "feves_me: ME launch: %s\n", cudaGetErrorString(e)); return ME_ECUDA; }
  tmark(c, 3, st);
  c->last_launches++;
  return launch_status();
}

static int launch_int(me_ctx* c, const uint8_t* rf, uint8_t* sf, cudaStream_t st) {
  IntParams P;
  P.rf = rf; P.sf = sf; P.W = c->W; P.H = c->H;
  P.k_hi = kAvgHi;
  P.pad = c->sf_pad; P.pitch = c->sf_pitch; P.rows = c->sf_rows;
  P.plane = (size_t)c->sf_rows * c->sf_pitch;
  if (c->row0 == 0 && c->row1 == c->mb_rows) {
    P.row_begin = 0; P.row_end = c->sf_rows;
  } else {   // stripe + halo: SME reads integer rows [16r0-R-1, 16r1+R-2]
    P.row_begin = std::max(0, c->sf_pad + 16 * c->row0 - c->R - c->max_pmv - 4);
    P.row_end = std::min(c->sf_rows, c->sf_pad + 16 * c->row1 + c->R + c->max_pmv + 4);
  }
  const int groups = c->sf_pitch / 16;
  // interior groups: x0-4 >= 0 and x0+20 <= W with x0 = 16g - pad, rows 4-byte aligned
  int g_lo = groups, g_hi = groups;
  if (c->W % 4 == 0 && (reinterpret_cast<uintptr_t>(rf) & 3) == 0) {
    g_lo = std::min(groups, (c->sf_pad + 4 + 15) / 16);
    g_hi = std::max(g_lo, std::min(groups, (c->W - 20 + c->sf_pad) / 16 + 1));
  }
  P.g_lo = g_lo; P.g_hi = g_hi;
  const int nb = groups - (g_hi - g_lo);
  int bx = 1;
  while (bx < nb && bx < 32) bx <<= 1;
  P.border_bx = bx;
  const int nrows = P.row_end - P.row_begin;
  P.vec_ok = (c->W % 4 == 0 && (reinterpret_cast<uintptr_t>(rf) & 3) == 0) ? 1 : 0;
  tmark(c, 0, st);
  if (c->int_kernel == 1) {   // shared-memory tiled (int_tile_kernel)
    const dim3 grid((groups + kIntTx - 1) / kIntTx, ((nrows + kIntTy - 1) / kIntTy + FEVES_INT_TPC - 1) / FEVES_INT_TPC);
    int_tile_kernel<<<grid, dim3(kIntTx, kIntTy), 0, st>>>(P);
  } else {                    // one thread per 16 columns x 1 row, global loads (int_subpel_kernel)
    const dim3 block(32, 4);
    // x: interior blocks of 32 groups, or the border slices of bx groups (z = 0), whichever is more
    const dim3 grid(std::max(std::max(1, (g_hi - g_lo + 31) / 32), (nb + bx - 1) / bx), (nrows + 3) / 4,
                    nb > 0 ? 2 : 1);
    int_subpel_kernel<<<grid, block, 0, st>>>(P);
  }
  c->last_launches++;
  tmark(c, 1, st);
  return launch_status();
}

static int launch_sme(me_ctx* c, const uint8_t* cf, const uint8_t* const* sfs, const int16_t* in_mvs,
                      const uint16_t* in_sads, int16_t* out_qmvs, uint16_t* out_sads, int n_ref, cudaStream_t st,
                      int rf0 = 0, int marks = 3) {   // marks: bit 0 = start timer event, bit 1 = stop
  SmeParams P;
  memset(&P, 0, sizeof(P));
  P.cf = cf;
  for (int k = 0; k < n_ref; ++k) P.sf[k] = sfs[k];
  P.in_mvs = reinterpret_cast<const uint32_t*>(in_mvs);
  P.in_sads = in_sads;
  P.out_qmvs = reinterpret_cast<uint32_t*>(out_qmvs);
  P.out_sads = out_sads;
  P.W = c->W; P.H = c->H; P.n_rf = n_ref; P.rf_stride = c->n_rf; P.mb_cols = c->mb_cols; P.row0 = c->row0;
  P.n_rows = c->row1 - c->row0;
  P.groups = (c->mb_cols + 7) / 8;
  P.lambda = c->lambda;
  P.pmv = c->d_pmv ? c->d_pmv + 2 * rf0 : nullptr;
  P.max_pmv = c->max_pmv;
  P.pad = c->sf_pad; P.pitch = c->sf_pitch;
  P.plane = (size_t)c->sf_rows * c->sf_pitch;
  P.fence = is_peer_ptr(c, out_qmvs) || is_peer_ptr(c, out_sads);
  P.cf_vec = (c->W % 4 == 0) && ((reinterpret_cast<uintptr_t>(cf) & 3) == 0);   // aligned CF word loads
  P.k_hi = kAvgHi;
  const int warps = n_ref * P.n_rows * P.groups;
  // SME work per warp (ME_OPT_SME_SPLIT): 1 = one mode (7 warps per MB group, all its partition
  // groups in turn), 2 = one partition group (16 warps), 3 = the 4-group modes as two warps of two
  // groups (9 warps); 0 (auto) = 3 when the grid would not fill the GPU ~6 times over, else 1.
  // 1080p S64 4 RF (tools/stripe_probe.py): whole frame 141.2 (1) / 143.4 (3) / 153.1 us (2);
  // 34-row stripe 80.9 (2) / 75.8 us (3); 9-row stripe 44.2 (1) / 33.8 (2) / 31.6 us (3)
  P.split = (c->sme_split == 3 || (c->sme_split == 0 && 7 * warps < c->sme_split_warps)) ? 3 : c->sme_split == 2 ? 1 : 0;
  if (marks & 1) tmark(c, 4, st);
  // shared-memory staged SME (sme_smem.cuh) for the SAD distortion with the ME SADs given
  // and 16-byte aligned SFs (cp.async); the global-load kernel otherwise
  bool staged = c->sme_kernel == 1 && !c->satd && in_sads != nullptr;
  for (int k = 0; k < n_ref; ++k) staged = staged && ((reinterpret_cast<uintptr_t>(sfs[k]) & 15) == 0);
  cudaError_t e;
  if (staged) {
    e = sme2_launch(c->lambda != 0, n_ref * P.n_rows * ((c->mb_cols + kSme2Mb - 1) / kSme2Mb), st, P, c->d_ovf);
    c->last_launches += 2;
  } else {
    const dim3 sg((warps + 3) / 4, P.split == 3 ? 9 : P.split ? 16 : 7);   // y = partition mode (or mode x groups)
    e = sme_launch(c->lambda != 0, c->satd != 0, sg, 128, st, P);
    c->last_launches++;
  }
  if (e != cudaSuccess) { fprintf(stderr, "feves_me: SME launch: %s\n", cudaGetErrorString(e)); return ME_ECUDA; }
  if (marks & 2) tmark(c, 5, st);
  return launch_status();
}

// ME then SME of n_ref RFs.  Pipelined (ME_OPT_PIPELINE_RF): one ME launch per RF on
// the compute stream, and the SME of RF k on the SME stream as soon as the ME of RF k
// is done (the only dependency), so the memory-latency-bound SME of RF k co-runs
// with the ALU-bound ME of RF k+1.  sf_ready (may be null) gates the first SME.
static int run_me_sme(me_ctx* c, const uint8_t* cf, const uint8_t* const* rfs, const uint8_t* const* sfs,
                      int16_t* mvs, uint16_t* sads, int16_t* qmvs, uint16_t* qsads, int n_ref, cudaEvent_t sf_ready) {
  int st;
  if (!c->pipeline) {
    if ((st = launch_me(c, cf, rfs, mvs, sads, n_ref, c->stream)) != ME_OK) return st;
    if (sf_ready && cudaStreamWaitEvent(c->stream, sf_ready, 0) != cudaSuccess) return launch_status();
    return launch_sme(c, cf, sfs, mvs, sads, qmvs, qsads, n_ref, c->stream);
  }
  if (!c->sme_st) {
    if (cudaStreamCreateWithFlags(&c->sme_st, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&c->ev_sme_done, cudaEventDisableTiming) != cudaSuccess)
      return launch_status();
    for (int k = 0; k < kMaxRf; ++k)
      if (cudaEventCreateWithFlags(&c->ev_me[k], cudaEventDisableTiming) != cudaSuccess) return launch_status();
  }
  const int saved = c->timing;
  c->timing = 0;   // per-module timers are not meaningful for interleaved launches
  // the SME stream must see everything enqueued on the compute stream so far
  if (cudaEventRecord(c->ev_sme_done, c->stream) != cudaSuccess ||
      cudaStreamWaitEvent(c->sme_st, c->ev_sme_done, 0) != cudaSuccess)
    return launch_status();
  if (sf_ready && cudaStreamWaitEvent(c->sme_st, sf_ready, 0) != cudaSuccess) return launch_status();
  for (int k = 0; k < n_ref; ++k) {
    const size_t off = (size_t)k * kNPart;
    if ((st = launch_me(c, cf, rfs + k, mvs + 2 * off, sads + off, 1, c->stream, nullptr, nullptr, nullptr, k)) != ME_OK)
      return st;
    if (cudaEventRecord(c->ev_me[k], c->stream) != cudaSuccess ||
        cudaStreamWaitEvent(c->sme_st, c->ev_me[k], 0) != cudaSuccess)
      return launch_status();
    if ((st = launch_sme(c, cf, sfs + k, mvs + 2 * off, sads + off, qmvs + 2 * off, qsads + off, 1, c->sme_st, k)) !=
        ME_OK)
      return st;
  }
  c->timing = saved;
  if (cudaEventRecord(c->ev_sme_done, c->sme_st) != cudaSuccess ||
      cudaStreamWaitEvent(c->stream, c->ev_sme_done, 0) != cudaSuccess)
    return launch_status();
  return ME_OK;
}

// ------------------------------------------------------------------ API ----
extern "C" int me_estimate(me_ctx* c, const uint8_t* cf, const uint8_t* const* rfs, int16_t* out_mvs,
                           uint16_t* out_sads) {
  if (!c || !rfs) return ME_EINVAL;
  if (!is_device_ptr(c, cf) || !is_device_ptr(c, out_mvs) || !is_device_ptr(c, out_sads)) return ME_EINVAL;
  for (int k = 0; k < c->n_rf; ++k)
    if (!is_device_ptr(c, rfs[k])) return ME_EINVAL;
  c->last_launches = 0;
  return launch_me(c, cf, rfs, out_mvs, out_sads, c->n_rf, c->stream);
}

extern "C" int int_interpolate(me_ctx* c, const uint8_t* rf, uint8_t* out_sf) {
  if (!c || !is_device_ptr(c, rf) || !is_device_ptr(c, out_sf)) return ME_EINVAL;
  c->last_launches = 0;
  return launch_int(c, rf, out_sf, c->stream);
}

extern "C" int sme_refine(me_ctx* c, const uint8_t* cf, const uint8_t* const* sfs, const int16_t* in_mvs,
                          const uint16_t* in_sads, int16_t* out_qmvs, uint16_t* out_sads) {
  if (!c || !sfs) return ME_EINVAL;
  if (!is_device_ptr(c, cf) || !is_device_ptr(c, in_mvs) || !is_device_ptr(c, out_qmvs) ||
      !is_device_ptr(c, out_sads))
    return ME_EINVAL;
  if (in_sads && !is_device_ptr(c, in_sads)) return ME_EINVAL;
  for (int k = 0; k < c->n_rf; ++k)
    if (!is_device_ptr(c, sfs[k])) return ME_EINVAL;
  c->last_launches = 0;
  return launch_sme(c, cf, sfs, in_mvs, in_sads, out_qmvs, out_sads, c->n_rf, c->stream);
}

extern "C" int me_encode_frame(me_ctx* c, const uint8_t* cf, const uint8_t* const* rfs, uint8_t* const* sfs,
                               int n_int, int16_t* out_mvs, uint16_t* out_sads, int16_t* out_qmvs,
                               uint16_t* out_qsads) {
  if (!c || !rfs || !sfs || n_int < 0 || n_int > c->n_rf) return ME_EINVAL;
  if (!is_device_ptr(c, cf) || !is_device_ptr(c, out_qmvs) || !is_device_ptr(c, out_qsads)) return ME_EINVAL;
  if ((out_mvs && !is_device_ptr(c, out_mvs)) || (out_sads && !is_device_ptr(c, out_sads))) return ME_EINVAL;
  for (int k = 0; k < c->n_rf; ++k)
    if (!is_device_ptr(c, rfs[k]) || !is_device_ptr(c, sfs[k])) return ME_EINVAL;
  int16_t* mvs = out_mvs ? out_mvs : c->d_mvs;
  uint16_t* sads = out_sads ? out_sads : c->d_sads;
  c->last_launches = 0;
  c->timed_mask = 0;
  int st;
  for (int k = 0; k < n_int; ++k)
    if ((st = launch_int(c, rfs[k], sfs[k], c->stream)) != ME_OK) return st;
  if (c->fuse && !c->lambda && !c->satd && !c->inclusive && !c->max_pmv)   // ME with the SME fused (one launch; base reading only)
    return launch_me(c, cf, rfs, out_mvs, out_sads, c->n_rf, c->stream, reinterpret_cast<const uint8_t* const*>(sfs),
                     out_qmvs, out_qsads);
  return run_me_sme(c, cf, rfs, reinterpret_cast<const uint8_t* const*>(sfs), mvs, sads, out_qmvs, out_qsads, c->n_rf,
                    nullptr);
}

// ------------------------------------------------------------ IPPP stream ----
// frames are encoded in order (frame t needs the RFs reconstructed from
// t-1, t-2, ...); the number of usable RFs ramps up over the first
// frames; "ME and INT can be simultaneously processed".  Here the RF of
// frame t-1 is the frame itself (no R* reconstruction on this path, DESIGN.md
// §9).  Push of frame t: copy it into ring slot t mod (n_rf+1); INT(frame t-1)
// into SF slot (t-1) mod n_rf on the side stream, concurrently with ME of frame
// t over its min(t, n_rf) RFs; join; SME; outputs (quarter-pel MVs + SADs).
extern "C" int me_stream_reset(me_ctx* c) {
  if (!c) return ME_EINVAL;
  c->t = 0;
  c->gepoch++;
  return ME_OK;
}

// ring of n_rf + 2 frames: the slot written by push t held frame t-n_rf-2, last
// read by the compute of push t-2, so the upload of t overlaps the compute of t-1
static int ring_slots(const me_ctx* c) { return c->n_rf + 2; }

static int stream_alloc(me_ctx* c) {
  if (c->ring) return ME_OK;
  const size_t fb = (size_t)c->W * c->H, sb = (size_t)kNPhase * c->sf_rows * c->sf_pitch;
  const size_t nmv = (size_t)c->mb_cols * c->mb_rows * c->n_rf * kNPart;
  bool ok = cudaMalloc(&c->ring, fb * ring_slots(c)) == cudaSuccess &&
            cudaMalloc(&c->sf_ring, sb * c->n_rf) == cudaSuccess && cudaMalloc(&c->d_qmvs, nmv * 4) == cudaSuccess &&
            cudaMalloc(&c->d_qsads, nmv * 2) == cudaSuccess &&
            cudaStreamCreateWithPriority(&c->side, cudaStreamNonBlocking, 0 /* lowest */) == cudaSuccess &&
            cudaStreamCreateWithFlags(&c->copy_in, cudaStreamNonBlocking) == cudaSuccess &&
            cudaStreamCreateWithFlags(&c->copy_out, cudaStreamNonBlocking) == cudaSuccess &&
            cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming) == cudaSuccess &&
            cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming) == cudaSuccess;
  for (int i = 0; ok && i < 2; ++i)
    ok = cudaEventCreateWithFlags(&c->ev_done[i], cudaEventDisableTiming) == cudaSuccess &&
         cudaEventCreateWithFlags(&c->ev_up[i], cudaEventDisableTiming) == cudaSuccess &&
         cudaEventCreateWithFlags(&c->ev_down[i], cudaEventDisableTiming) == cudaSuccess &&
         cudaMalloc(&c->d_qmvs2[i], nmv * 4) == cudaSuccess && cudaMalloc(&c->d_qsads2[i], nmv * 2) == cudaSuccess &&
         cudaEventRecord(c->ev_done[i], c->stream) == cudaSuccess &&     // "already done" for t < 2
         cudaEventRecord(c->ev_down[i], c->stream) == cudaSuccess;
  if (!ok) {
    cudaGetLastError();
    return ME_ENOMEM;
  }
  return ME_OK;
}

// ME_OPT_OVERLAP_SME: push t enqueues
//   side : wait(main fork), wait(SME(t-1) done)   INT(t-1) -> SF slot (t-1) mod n_rf
//          (that slot held frame t-1-n_rf, which SME(t-1) read as its last RF)
//   main : ME(t) -> ME buffer t & 1; then wait(SME(t-1) done), so everything later on the
//          context stream (the next frame copy, ME(t+1), the caller) sees frame t-1 complete
//   ov_st: wait(ME(t)), wait(INT(t-1))             SME(t) -> outputs
// so SME(t) (latency-bound) co-runs with ME(t+1) (ALU-bound) of the next push.  The ME
// outputs are double-buffered because ME(t+1) writes while SME(t) reads.
static int push_overlapped(me_ctx* c, const uint8_t* cur, const uint8_t* const* rfs, const uint8_t* const* sfs,
                           const uint8_t* new_rf, uint8_t* new_sf, int16_t* qm, uint16_t* qs, int n_ref, int par) {
  if (!c->ov_st) {
    int lo = 0, hi = 0;
    const size_t nmv = (size_t)c->mb_cols * c->mb_rows * c->n_rf * kNPart;
    bool ok = cudaDeviceGetStreamPriorityRange(&lo, &hi) == cudaSuccess &&
              cudaStreamCreateWithPriority(&c->ov_st, cudaStreamNonBlocking, hi) == cudaSuccess &&
              cudaEventCreateWithFlags(&c->ev_ov_me, cudaEventDisableTiming) == cudaSuccess &&
              cudaEventCreateWithFlags(&c->ev_ov_sme, cudaEventDisableTiming) == cudaSuccess;
    for (int i = 0; ok && i < 2; ++i)
      ok = cudaMalloc(&c->d_mvs_ov[i], nmv * 4) == cudaSuccess && cudaMalloc(&c->d_sads_ov[i], nmv * 2) == cudaSuccess;
    if (!ok) { cudaGetLastError(); return ME_ENOMEM; }
  }
  int st;
  if (cudaEventRecord(c->ev_fork, c->stream) != cudaSuccess ||
      cudaStreamWaitEvent(c->side, c->ev_fork, 0) != cudaSuccess ||
      (c->ov_pending && cudaStreamWaitEvent(c->side, c->ev_ov_sme, 0) != cudaSuccess))
    return launch_status();
  if ((st = launch_int(c, new_rf, new_sf, c->side)) != ME_OK) return st;
  if (cudaEventRecord(c->ev_join, c->side) != cudaSuccess) return launch_status();
  if ((st = launch_me(c, cur, rfs, c->d_mvs_ov[par], c->d_sads_ov[par], n_ref, c->stream)) != ME_OK) return st;
  if (cudaEventRecord(c->ev_ov_me, c->stream) != cudaSuccess ||
      (c->ov_pending && cudaStreamWaitEvent(c->stream, c->ev_ov_sme, 0) != cudaSuccess) ||
      cudaStreamWaitEvent(c->ov_st, c->ev_ov_me, 0) != cudaSuccess ||
      cudaStreamWaitEvent(c->ov_st, c->ev_join, 0) != cudaSuccess)
    return launch_status();
  if ((st = launch_sme(c, cur, sfs, c->d_mvs_ov[par], c->d_sads_ov[par], qm, qs, n_ref, c->ov_st)) != ME_OK) return st;
  if (cudaEventRecord(c->ev_ov_sme, c->ov_st) != cudaSuccess) return launch_status();
  c->ov_pending = true;
  return ME_OK;
}

// The enqueue body of me_stream_push (arguments validated, ring allocated).
static int push_enqueue(me_ctx* c, const uint8_t* cf, int cf_on_host, int16_t* out_qmvs, uint16_t* out_qsads,
                        int out_on_host, int* n_ref_used) {
  int st;
  c->last_launches = 0;
  c->timed_mask = 0;
  const size_t fb = (size_t)c->W * c->H, sb = (size_t)kNPhase * c->sf_rows * c->sf_pitch;
  const int slots = ring_slots(c);
  const long long t = c->t;
  const int par = (int)(t & 1);
  uint8_t* cur = c->ring + (size_t)(t % slots) * fb;
  // rows of every frame this stripe reads (ME +-R, SME +1, 6-tap -2..+3)
  int y0 = 0, y1 = c->H;
  if (c->halo_only) {
    y0 = std::max(0, 16 * c->row0 - c->R - c->max_pmv - 6);   // + the predictor's reach (G21)
    y1 = std::min(c->H, 16 * c->row1 + c->R + c->max_pmv + 7);
  }
  const int n_ref = (int)std::min<long long>(t, c->n_rf);
  for (int k = 0; k < n_ref; ++k) {             // a re-split may need rows a halo-only frame lacks
    const int s = (int)((t - 1 - k) % slots);
    if (c->fv0[s] > y0 || c->fv1[s] < y1) return ME_ESTATE;
  }
  const size_t off = (size_t)y0 * c->W, len = (size_t)(y1 - y0) * c->W;
  if (cf_on_host || c->wait_flag) {
    // upload (host frame) / pull (device or peer frame published with a flag) on the copy-in
    // stream once the compute of push t-2 (last reader of this slot) is done, so it overlaps the
    // compute of push t-1 (P:51 copy engines; SURVEY §8(e) frame t+1 under frame t's compute)
    if (cudaStreamWaitEvent(c->copy_in, c->ev_done[par], 0) != cudaSuccess) return launch_status();
    if (c->wait_flag && (st = stream_wait_value(c->copy_in, c->wait_flag, c->wait_value)) != ME_OK) return st;
    if (cudaMemcpyAsync(cur + off, cf + off, len, cf_on_host ? cudaMemcpyHostToDevice : cudaMemcpyDefault,
                        c->copy_in) != cudaSuccess ||
        cudaEventRecord(c->ev_up[par], c->copy_in) != cudaSuccess ||
        cudaStreamWaitEvent(c->stream, c->ev_up[par], 0) != cudaSuccess)
      return launch_status();
  } else if (cudaMemcpyAsync(cur + off, cf + off, len, cudaMemcpyDefault, c->stream) != cudaSuccess) {
    return launch_status();   // (cudaMemcpyDefault: cf may be a peer GPU's buffer, me_ipc_open)
  }
  c->fv0[t % slots] = y0;
  c->fv1[t % slots] = y1;
  if (n_ref_used) *n_ref_used = n_ref;
  if (n_ref > 0) {
    uint8_t* new_rf = c->ring + (size_t)((t - 1) % slots) * fb;
    uint8_t* new_sf = c->sf_ring + (size_t)((t - 1) % c->n_rf) * sb;
    const uint8_t* rfs[kMaxRf];
    const uint8_t* sfs[kMaxRf];
    for (int k = 0; k < n_ref; ++k) {           // ref_idx k = frame t-1-k
      rfs[k] = c->ring + (size_t)((t - 1 - k) % slots) * fb;
      sfs[k] = c->sf_ring + (size_t)((t - 1 - k) % c->n_rf) * sb;
    }
    // f3 re-split: an SF computed for another stripe may lack rows this stripe reads;
    // recompute it from the frame ring (the ring holds whole frames) before ME/SME
    for (int k = 1; k < n_ref; ++k) {
      const int slot = (int)((t - 1 - k) % c->n_rf);
      if (!(c->sf_v0[slot] <= c->row0 && c->row1 <= c->sf_v1[slot])) {
        if ((st = launch_int(c, rfs[k], c->sf_ring + (size_t)slot * sb, c->stream)) != ME_OK) return st;
        c->sf_v0[slot] = c->row0;
        c->sf_v1[slot] = c->row1;
      }
    }
    {
      const int slot = (int)((t - 1) % c->n_rf);   // INT of the newest RF below covers this stripe
      c->sf_v0[slot] = c->row0;
      c->sf_v1[slot] = c->row1;
    }
    int16_t* qm = (out_qmvs && !out_on_host) ? out_qmvs : (out_on_host ? c->d_qmvs2[par] : c->d_qmvs);
    uint16_t* qs = (out_qsads && !out_on_host) ? out_qsads : (out_on_host ? c->d_qsads2[par] : c->d_qsads);
    // the device output buffer t & 1 is free once the download of push t-2 finished
    if (out_on_host && cudaStreamWaitEvent(c->stream, c->ev_down[par], 0) != cudaSuccess) return launch_status();
    if (c->overlap && !c->pipeline && !(c->fuse && !c->lambda && !c->satd && !c->inclusive && !c->max_pmv)) {
      if ((st = push_overlapped(c, cur, rfs, sfs, new_rf, new_sf, qm, qs, n_ref, par)) != ME_OK) return st;
    } else if (c->fuse && !c->lambda && !c->satd && !c->inclusive && !c->max_pmv) {
      // fused: the SME of ref 0 reads SF(t-1), so INT(t-1) runs first on the same stream
      if ((st = launch_int(c, new_rf, new_sf, c->stream)) != ME_OK) return st;
      if ((st = launch_me(c, cur, rfs, nullptr, nullptr, n_ref, c->stream, sfs, qm, qs)) != ME_OK) return st;
    } else {
      // side stream: INT of the newest RF (frame t-1), concurrent with ME
      if (cudaEventRecord(c->ev_fork, c->stream) != cudaSuccess ||
          cudaStreamWaitEvent(c->side, c->ev_fork, 0) != cudaSuccess)
        return launch_status();
      if ((st = launch_int(c, new_rf, new_sf, c->side)) != ME_OK) return st;
      if (cudaEventRecord(c->ev_join, c->side) != cudaSuccess) return launch_status();
      if ((st = run_me_sme(c, cur, rfs, sfs, c->d_mvs, c->d_sads, qm, qs, n_ref, c->ev_join)) != ME_OK) return st;
    }
    const size_t nmv = (size_t)(c->row1 - c->row0) * c->mb_cols * c->n_rf * kNPart;
    if (c->signal_flag && (st = stream_write_value(c->ov_pending ? c->ov_st : c->stream, c->signal_flag,
                                                   c->signal_value)) != ME_OK)
      return st;
    if (cudaEventRecord(c->ev_done[par], c->ov_pending ? c->ov_st : c->stream) != cudaSuccess) return launch_status();
    if (out_on_host) {   // download on the copy-out stream, overlapping the next frame's compute
      // only the n_ref searched RF slots of every MB (slots >= n_ref stay untouched, as for
      // device outputs): one 2-D copy, rows = MBs, pitch = n_rf slots
      const size_t n_mb = nmv / ((size_t)c->n_rf * kNPart), slot = (size_t)kNPart;
      const size_t pm = (size_t)c->n_rf * slot * 4, ps = (size_t)c->n_rf * slot * 2;
      if (cudaStreamWaitEvent(c->copy_out, c->ev_done[par], 0) != cudaSuccess ||
          (out_qmvs && cudaMemcpy2DAsync(out_qmvs, pm, qm, pm, (size_t)n_ref * slot * 4, n_mb, cudaMemcpyDeviceToHost,
                                         c->copy_out) != cudaSuccess) ||
          (out_qsads && cudaMemcpy2DAsync(out_qsads, ps, qs, ps, (size_t)n_ref * slot * 2, n_mb, cudaMemcpyDeviceToHost,
                                          c->copy_out) != cudaSuccess) ||
          cudaEventRecord(c->ev_down[par], c->copy_out) != cudaSuccess)
        return launch_status();
    }
  } else {
    if (c->signal_flag && (st = stream_write_value(c->stream, c->signal_flag, c->signal_value)) != ME_OK) return st;
    if (cudaEventRecord(c->ev_done[par], c->stream) != cudaSuccess) return launch_status();
  }
  c->t = t + 1;
  return ME_OK;
}

// ME_OPT_GRAPH: a device-resident steady-state push (all n_rf RFs present, device frame and
// outputs, no SF refresh pending) is captured once per ring phase into a CUDA graph and
// replayed afterwards (SURVEY §8(d) "one CUDA graph per frame").  The ring / SF slots a
// push uses repeat with period lcm(n_rf + 2, n_rf, 2) (frame ring, SF ring, output parity);
// a graph is keyed by its phase and the caller's pointers and dropped when any setting
// changes (gepoch).  The host-side ring bookkeeping of a replayed push is the same as the
// captured one's, so it is replayed on the host alongside the graph.
static int graph_period(const me_ctx* c) {
  auto gcd = [](int a, int b) { while (b) { const int t = a % b; a = b; b = t; } return a; };
  const int a = ring_slots(c), b = c->n_rf, l = a / gcd(a, b) * b;
  return l / gcd(l, 2) * 2;
}

static bool push_needs_sf_refresh(const me_ctx* c) {
  for (int k = 1; k < c->n_rf; ++k) {
    const int slot = (int)((c->t - 1 - k) % c->n_rf);
    if (!(c->sf_v0[slot] <= c->row0 && c->row1 <= c->sf_v1[slot])) return true;
  }
  return false;
}

static int push_graph(me_ctx* c, const uint8_t* cf, int16_t* out_qmvs, uint16_t* out_qsads, int* n_ref_used,
                      int period);

extern "C" int me_stream_push(me_ctx* c, const uint8_t* cf, int cf_on_host, int16_t* out_qmvs,
                              uint16_t* out_qsads, int out_on_host, int* n_ref_used) {
  if (!c || !cf) return ME_EINVAL;
  if (!cf_on_host && !is_device_ptr(c, cf)) return ME_EINVAL;
  if (out_qmvs && !out_on_host && !is_device_ptr(c, out_qmvs)) return ME_EINVAL;
  if (out_qsads && !out_on_host && !is_device_ptr(c, out_qsads)) return ME_EINVAL;
  int st = stream_alloc(c);
  if (st != ME_OK) return st;
  const int period = graph_period(c);
  const bool graph = c->graph && !cf_on_host && !out_on_host && !c->overlap && !c->pipeline && !c->fuse &&
                     !c->wait_flag && !c->signal_flag &&
                     c->t >= c->n_rf && period <= 64 && !push_needs_sf_refresh(c);
  if (!graph) return push_enqueue(c, cf, cf_on_host, out_qmvs, out_qsads, out_on_host, n_ref_used);
  return push_graph(c, cf, out_qmvs, out_qsads, n_ref_used, period);
}

static int push_graph(me_ctx* c, const uint8_t* cf, int16_t* out_qmvs, uint16_t* out_qsads, int* n_ref_used,
                      int period) {
  int st;
  if ((int)c->graphs.size() != period) { graphs_drop(c); c->graphs.resize(period); }
  me_ctx::Graph& g = c->graphs[c->t % period];
  const long long t = c->t;
  const int par = (int)(t & 1);
  const int slots = ring_slots(c);
  if (g.exec && g.qm == out_qmvs && g.qs == out_qsads && g.row0 == c->row0 && g.row1 == c->row1 &&
      g.epoch == c->gepoch && g.timing == c->timing) {
    // replay: the host bookkeeping push_enqueue did when this phase was captured
    int y0 = 0, y1 = c->H;
    if (c->halo_only) {
      y0 = std::max(0, 16 * c->row0 - c->R - c->max_pmv - 6);
      y1 = std::min(c->H, 16 * c->row1 + c->R + c->max_pmv + 7);
    }
    for (int k = 0; k < c->n_rf; ++k) {
      const int s = (int)((t - 1 - k) % slots);
      if (c->fv0[s] > y0 || c->fv1[s] < y1) return ME_ESTATE;
    }
    if (g.cf != cf) {                                 // this push's frame: re-point the copy node
      const size_t off = (size_t)y0 * c->W, len = (size_t)(y1 - y0) * c->W;
      uint8_t* cur = c->ring + (size_t)(t % slots) * ((size_t)c->W * c->H);
      if (cudaGraphExecMemcpyNodeSetParams1D(g.exec, g.copy, cur + off, cf + off, len, cudaMemcpyDefault) !=
          cudaSuccess)
        return launch_status();
      g.cf = cf;
    }
    if (cudaGraphLaunch(g.exec, c->stream) != cudaSuccess ||
        cudaEventRecord(c->ev_done[par], c->stream) != cudaSuccess)
      return launch_status();
    c->fv0[t % slots] = y0;
    c->fv1[t % slots] = y1;
    const int slot = (int)((t - 1) % c->n_rf);
    c->sf_v0[slot] = c->row0;
    c->sf_v1[slot] = c->row1;
    c->last_launches = g.launches;
    c->timed_mask = g.timed_mask;
    c->t = t + 1;
    if (n_ref_used) *n_ref_used = c->n_rf;
    return ME_OK;
  }
  // capture this phase on the context's own stream (capturable even when the caller's is the
  // legacy default stream; nothing executes during a capture, so no ordering is needed), then
  // launch it on the caller's stream (the timers become external event-record nodes, tmark)
  cudaStream_t caller = c->stream;
  c->stream = c->own;
  if (cudaStreamBeginCapture(c->stream, cudaStreamCaptureModeThreadLocal) != cudaSuccess) {
    c->stream = caller;
    return launch_status();
  }
  c->capturing = true;
  st = push_enqueue(c, cf, 0, out_qmvs, out_qsads, 0, n_ref_used);
  c->capturing = false;
  cudaGraph_t gr = nullptr;
  const cudaError_t ec = cudaStreamEndCapture(c->stream, &gr);
  c->stream = caller;
  if (st != ME_OK || ec != cudaSuccess) {
    if (gr) cudaGraphDestroy(gr);
    cudaGetLastError();
    return st != ME_OK ? st : ME_ECUDA;
  }
  if (g.exec) { cudaGraphExecDestroy(g.exec); g.exec = nullptr; }
  if (g.graph) { cudaGraphDestroy(g.graph); g.graph = nullptr; }
  g.copy = nullptr;
  size_t nn = 0;
  cudaGraphGetNodes(gr, nullptr, &nn);
  std::vector<cudaGraphNode_t> nodes(nn);
  cudaGraphGetNodes(gr, nodes.data(), &nn);
  for (cudaGraphNode_t n : nodes) {
    cudaGraphNodeType ty;
    if (cudaGraphNodeGetType(n, &ty) == cudaSuccess && ty == cudaGraphNodeTypeMemcpy) g.copy = n;
  }
  const cudaError_t ei = g.copy ? cudaGraphInstantiate(&g.exec, gr, cudaGraphInstantiateFlagUseNodePriority) : cudaErrorUnknown;
  if (ei != cudaSuccess) {
    g.exec = nullptr;
    cudaGraphDestroy(gr);
    cudaGetLastError();
    fprintf(stderr, "feves_me: stream graph: %s\n", cudaGetErrorString(ei));
    return ME_ECUDA;
  }
  g.graph = gr;
  g.cf = cf; g.qm = out_qmvs; g.qs = out_qsads; g.row0 = c->row0; g.row1 = c->row1;
  g.epoch = c->gepoch; g.timing = c->timing; g.launches = c->last_launches; g.timed_mask = c->timed_mask;
  if (cudaGraphLaunch(g.exec, c->stream) != cudaSuccess ||
      cudaEventRecord(c->ev_done[par], c->stream) != cudaSuccess)   // a real record (the captured one is a node)
    return launch_status();
  return ME_OK;
}

extern "C" int me_stream_push_flags(me_ctx* c, const uint8_t* cf, int cf_on_host, int16_t* out_qmvs,
                                    uint16_t* out_qsads, int out_on_host, int* n_ref_used, const uint32_t* wait_flag,
                                    uint32_t wait_value, uint32_t* signal_flag, uint32_t signal_value) {
  if (!c) return ME_EINVAL;
  if ((wait_flag && !is_device_ptr(c, wait_flag)) || (signal_flag && !is_device_ptr(c, signal_flag))) return ME_EINVAL;
  c->wait_flag = wait_flag; c->wait_value = wait_value;
  c->signal_flag = signal_flag; c->signal_value = signal_value;
  const int st = me_stream_push(c, cf, cf_on_host, out_qmvs, out_qsads, out_on_host, n_ref_used);
  c->wait_flag = nullptr; c->signal_flag = nullptr;
  return st;
}

extern "C" int me_stream_wait_value(void* stream, const uint32_t* flag, uint32_t value) {
  if (!flag) return ME_EINVAL;
  return stream_wait_value(reinterpret_cast<cudaStream_t>(stream), flag, value);
}

extern "C" int me_stream_write_value(void* stream, uint32_t* flag, uint32_t value) {
  if (!flag) return ME_EINVAL;
  return stream_write_value(reinterpret_cast<cudaStream_t>(stream), flag, value);
}

extern "C" int me_sync(me_ctx* c) {
  if (!c) return ME_EINVAL;
  cudaError_t e = cudaStreamSynchronize(c->stream);
  if (e == cudaSuccess && c->copy_in) e = cudaStreamSynchronize(c->copy_in);
  if (e == cudaSuccess && c->copy_out) e = cudaStreamSynchronize(c->copy_out);
  if (e == cudaSuccess && c->side) e = cudaStreamSynchronize(c->side);
  if (e == cudaSuccess && c->sme_st) e = cudaStreamSynchronize(c->sme_st);
  if (e == cudaSuccess && c->ov_st) e = cudaStreamSynchronize(c->ov_st);
  return e == cudaSuccess ? ME_OK : ME_ECUDA;
}

// the context stream waits for everything enqueued so far on the internal streams (copy-in,
// copy-out, INT side stream, SME streams): an event recorded on the context stream after this
// marks the end of all work of the pushes so far, including the last host download
extern "C" int me_stream_join(me_ctx* c) {
  if (!c) return ME_EINVAL;
  for (cudaStream_t s : {c->copy_in, c->copy_out, c->side, c->sme_st, c->ov_st}) {
    if (!s) continue;
    if (!c->ev_switch && cudaEventCreateWithFlags(&c->ev_switch, cudaEventDisableTiming) != cudaSuccess)
      return launch_status();
    if (cudaEventRecord(c->ev_switch, s) != cudaSuccess || cudaStreamWaitEvent(c->stream, c->ev_switch, 0) != cudaSuccess)
      return launch_status();
  }
  return ME_OK;
}

extern "C" int me_stream_outputs(me_ctx* c, int16_t** qmvs, uint16_t** qsads) {
  if (!c) return ME_EINVAL;
  if (qmvs) *qmvs = c->d_qmvs;
  if (qsads) *qsads = c->d_qsads;
  return ME_OK;
}

extern "C" int me_set_timing(me_ctx* c, int on) {
  if (!c) return ME_EINVAL;
  if (on && !c->ev_t[0])
    for (int i = 0; i < 6; ++i)
      if (cudaEventCreate(&c->ev_t[i]) != cudaSuccess) { cudaGetLastError(); return ME_ENOMEM; }
  if (c->timing != (on ? 1 : 0)) c->gepoch++;           // captured stream graphs hold the timer nodes
  c->timing = on ? 1 : 0;
  return ME_OK;
}

extern "C" int me_get_timings(me_ctx* c, float* ms_int, float* ms_me, float* ms_sme) {
  if (!c || !c->ev_t[0]) return ME_EINVAL;
  float* out[3] = {ms_int, ms_me, ms_sme};
  for (int k = 0; k < 3; ++k) {
    if (!out[k]) continue;
    *out[k] = -1.f;
    if (!(c->timed_mask & (1 << k))) continue;
    if (cudaEventSynchronize(c->ev_t[2 * k + 1]) != cudaSuccess ||
        cudaEventElapsedTime(out[k], c->ev_t[2 * k], c->ev_t[2 * k + 1]) != cudaSuccess)
      return launch_status();
  }
  return ME_OK;
}

extern "C" int me_set_option(me_ctx* c, int option, int value) {
  if (!c) return ME_EINVAL;
  c->gepoch++;                                          // cached stream graphs are stale
  switch (option) {
    case ME_OPT_GRAPH: c->graph = value ? 1 : 0; return ME_OK;
    case ME_OPT_INT_KERNEL:
      if (value < 0 || value > 1) return ME_EINVAL;
      c->int_kernel = value;
      return ME_OK;
    case ME_OPT_SME_SPLIT:
      if (value < 0 || value > 3) return ME_EINVAL;
      c->sme_split = value;
      return ME_OK;
    case ME_OPT_RF_PER_CTA:
      if (value < -1 || value > kMaxRf) return ME_EINVAL;
      c->rf_per_cta = value;
      return ME_OK;
    case ME_OPT_SME_KERNEL:
      if (value < 0 || value > 1) return ME_EINVAL;
      c->sme_kernel = value;
      return ME_OK;
    case ME_OPT_FUSED_SME: c->fuse = value ? 1 : 0; return ME_OK;
    case ME_OPT_PIPELINE_RF: c->pipeline = value ? 1 : 0; return ME_OK;
    case ME_OPT_ME_CTAS_PER_SM:
      if (value < 0 || value > 32) return ME_EINVAL;
      c->me_ctas_per_sm = value;
      return ME_OK;
    case ME_OPT_SA_INCLUSIVE:
      if (c->lambda > lambda_limit(c->S, value ? 1 : 0)) return ME_EINVAL;   // 32-bit key (see lambda_limit)
      if (c->stream) cudaStreamSynchronize(c->stream);   // the tables may be in use
      c->inclusive = value ? 1 : 0;
      return upload_key_table(c);
    case ME_OPT_SME_SATD:
      c->satd = value ? 1 : 0;
      return ME_OK;
    case ME_OPT_HALO_ONLY:
      c->halo_only = value ? 1 : 0;
      return ME_OK;
    case ME_OPT_OVERLAP_SME:
      if (c->stream) cudaStreamSynchronize(c->stream);
      if (c->ov_st) cudaStreamSynchronize(c->ov_st);
      c->ov_pending = false;
      c->overlap = value ? 1 : 0;
      return ME_OK;
    case ME_OPT_LAMBDA:
      if (value < 0 || value > lambda_limit(c->S, c->inclusive)) return ME_EINVAL;   // 32-bit key
      if (c->stream) cudaStreamSynchronize(c->stream);   // the table may be in use
      c->lambda = value;
      return upload_key_table(c);
    default: return ME_EINVAL;
  }
}

// ------------------------------------------------------------ peer memory ----
// stripe inputs and outputs move over NVLink by loads/stores of the
// kernels and copy engines instead of broadcast/gather collectives.
static int alloc_base(const void* p, uintptr_t* base) {
  using AddrRange = CUresult (*)(CUdeviceptr*, size_t*, CUdeviceptr);
  static AddrRange fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) != cudaSuccess || !f ||
        q != cudaDriverEntryPointSuccess) {
      cudaGetLastError();
      return ME_ECUDA;
    }
    fn = reinterpret_cast<AddrRange>(f);
  }
  CUdeviceptr b = 0;
  size_t sz = 0;
  if (fn(&b, &sz, reinterpret_cast<CUdeviceptr>(p)) != CUDA_SUCCESS) return ME_EINVAL;
  *base = static_cast<uintptr_t>(b);
  return ME_OK;
}

extern "C" int me_ipc_export(me_ctx* c, const void* dptr, void* handle, size_t* offset) {
  if (!c || !handle || !offset || !is_device_ptr(c, dptr)) return ME_EINVAL;
  for (int i = 0; i < c->n_peers; ++i)   // only this device's own allocations can be exported
    if (reinterpret_cast<uintptr_t>(dptr) >= c->peers[i].lo && reinterpret_cast<uintptr_t>(dptr) < c->peers[i].hi)
      return ME_EINVAL;
  uintptr_t base = 0;
  int st = alloc_base(dptr, &base);
  if (st != ME_OK) return st;
  cudaIpcMemHandle_t h;
  if (cudaIpcGetMemHandle(&h, reinterpret_cast<void*>(base)) != cudaSuccess) {
    cudaGetLastError();
    return ME_ECUDA;
  }
  static_assert(sizeof(h) == ME_IPC_HANDLE_BYTES, "CUDA IPC handle size");
  std::memcpy(handle, &h, sizeof(h));
  *offset = reinterpret_cast<uintptr_t>(dptr) - base;
  return ME_OK;
}

extern "C" int me_ipc_open(me_ctx* c, const void* handle, size_t offset, size_t bytes, void** dptr) {
  if (!c || !handle || !dptr || bytes == 0) return ME_EINVAL;
  int slot = -1;
  for (int i = 0; i < c->n_peers; ++i)
    if (!c->peers[i].base) { slot = i; break; }
  if (slot < 0) {
    if (c->n_peers == 16) return ME_EINVAL;
    slot = c->n_peers++;
  }
  cudaIpcMemHandle_t h;
  std::memcpy(&h, handle, sizeof(h));
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || (dev != c->device && cudaSetDevice(c->device) != cudaSuccess)) {
    cudaGetLastError();
    return ME_ECUDA;
  }
  void* base = nullptr;
  const cudaError_t e = cudaIpcOpenMemHandle(&base, h, cudaIpcMemLazyEnablePeerAccess);
  if (dev != c->device) cudaSetDevice(dev);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return e == cudaErrorInvalidValue || e == cudaErrorInvalidResourceHandle ? ME_EINVAL : ME_ECUDA;
  }
  const uintptr_t lo = reinterpret_cast<uintptr_t>(base) + offset;
  c->peers[slot] = {lo, lo + bytes, base};
  *dptr = reinterpret_cast<void*>(lo);
  return ME_OK;
}

extern "C" int me_ipc_close(me_ctx* c, void* dptr) {
  if (!c || !dptr) return ME_EINVAL;
  for (int i = 0; i < c->n_peers; ++i)
    if (c->peers[i].base && c->peers[i].lo == reinterpret_cast<uintptr_t>(dptr)) {
      if (c->stream) cudaStreamSynchronize(c->stream);   // kernels may still use it
      const cudaError_t e = cudaIpcCloseMemHandle(c->peers[i].base);
      c->peers[i] = {0, 0, nullptr};
      return e == cudaSuccess ? ME_OK : ME_ECUDA;
    }
  return ME_EINVAL;
}

extern "C" int me_sme_overflow_count(me_ctx* c) {
  if (!c) return ME_EINVAL;
  int n = 0;
  if (cudaStreamSynchronize(c->stream) != cudaSuccess ||
      cudaMemcpy(&n, c->d_ovf, sizeof(int), cudaMemcpyDeviceToHost) != cudaSuccess)
    return launch_status();
  return n;
}

extern "C" int me_set_fused(me_ctx* c, int on) { return me_set_option(c, ME_OPT_FUSED_SME, on); }

extern "C" int me_set_pmv(me_ctx* c, const int16_t* pmv) {
  if (!c) return ME_EINVAL;
  if (c->max_pmv == 0) return ME_ESTATE;               // the SF margin has no room for a predictor
  if (pmv && !is_device_ptr(c, pmv)) return ME_EINVAL;
  c->d_pmv = pmv;
  c->gepoch++;
  return ME_OK;
}

extern "C" int me_mode_decision(me_ctx* c, const int16_t* qmvs, const uint16_t* qsads, int n_ref, int32_t* out_modes) {
  if (!c || n_ref < 1 || n_ref > c->n_rf) return ME_EINVAL;
  if (!is_device_ptr(c, qmvs) || !is_device_ptr(c, qsads) || !is_device_ptr(c, out_modes)) return ME_EINVAL;
  ModeParams P;
  P.qmvs = reinterpret_cast<const uint32_t*>(qmvs);
  P.sads = qsads;
  P.out = out_modes;
  P.n_mb = (c->row1 - c->row0) * c->mb_cols;
  P.n_rf = n_ref;
  P.rf_stride = c->n_rf;
  P.lambda = c->lambda;
  P.pmv = c->d_pmv; P.max_pmv = c->max_pmv; P.mb0 = c->row0 * c->mb_cols;
  c->last_launches = 0;
  mode_decision_kernel<<<(P.n_mb + 127) / 128, 128, 0, c->stream>>>(P);
  c->last_launches++;
  return launch_status();
}
